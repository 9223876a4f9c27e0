// layout.h — compiled ALT layouts (product side).
//
// A layout is a row-major logical tensor transformed by a sequence of ALT
// layout primitives (paper §4.1, Table 1; unfold §4.1.2 P:727-749;
// pad P:783-786).  alt_layout_create compiles the sequence once into:
//   * the physical shape and row-major strides;
//   * a POD descriptor (LayoutDesc) that device code can interpret for any
//     layout (generic G / F evaluation, used by the fallback kernels);
//   * for SEPARABLE layouts (every physical dim derives from exactly one
//     logical dim — all split / reorder / pad / unfold sequences, and fuses
//     that stay inside one logical dim) per-logical-dim tables:
//       rd[d][i]     owner offset contribution of logical index i along d
//                    (physical offset = sum_d rd[d][i_d]);
//       rev[d][c]    logical index held by the c-th combination of d's
//                    physical coordinates (mixed radix), or -(clamped+1)
//                    for a structural zero (pad / unfold overhang);
//       wptr/wlist   every physical position "owned" by logical index i
//                    (its copies, plus the zero positions whose clamped
//                    owner is i), encoded as 2*offset + is_zero — this is
//                    what lets an epilogue write any layout directly
//                    (Fig. 5b);
//   * an affine descriptor when the raw map is affine: i_d = sum_p coef_p
//     j_p + off_d (used to cut TMA boxes out of the layout).
#pragma once
#include <cstdint>
#include <mutex>
#include <vector>

#include "alt.h"

namespace alt {

constexpr int kStageRank = 12;  // intermediate ranks during compilation
constexpr int kMaxL = 8;        // logical rank
constexpr int kMaxP = 10;       // physical rank

// POD copy of a compiled layout for the generic device interpreter.
struct LayoutDesc {
  int32_t lrank, np, prank, _pad;
  int32_t kind[ALT_MAX_PRIMS], dim[ALT_MAX_PRIMS], n[ALT_MAX_PRIMS];
  int64_t v[ALT_MAX_PRIMS][10];
  int32_t rank[ALT_MAX_PRIMS + 1];
  int64_t shp[ALT_MAX_PRIMS + 1][kStageRank];
  int64_t pstride[kMaxP];
};

// Device pointers of the separable tables (one blob per device).
struct SepDev {
  const int64_t *rd[kMaxL];
  const int32_t *rev[kMaxL];
  const int32_t *wptr[kMaxL];
  const int64_t *wlist[kMaxL];
};

struct Affine {
  bool ok = false;
  // per physical dim: owning logical dim and coefficient of the raw map
  int32_t pd[kMaxP];
  int64_t coef[kMaxP];
  // per logical dim: raw offset (i_d = sum coef_p j_p + off[d])
  int64_t off[kMaxL];
};

struct Layout {
  uint64_t serial = 0;  // unique per created layout (plan-cache keys)
  int32_t lrank = 0;
  int64_t lshape[kMaxL] = {};
  int32_t np = 0;
  alt_prim prims[ALT_MAX_PRIMS] = {};
  int32_t prank = 0;
  int64_t pshape[kMaxP] = {};
  int64_t pstride[kMaxP] = {};
  int64_t pnumel = 0, lnumel = 0;
  uint32_t flags = 0;
  LayoutDesc desc{};

  // separable description
  bool separable = false;
  int32_t pdim_owner[kMaxP] = {};   // logical dim of each physical dim
  int32_t pdim_rad[kMaxP] = {};     // mixed radix inside its logical dim
  int32_t footprint[kMaxL] = {};    // prod of extents of d's physical dims
  std::vector<int64_t> rd[kMaxL];
  std::vector<int32_t> rev[kMaxL];
  std::vector<int32_t> wptr[kMaxL];
  std::vector<int64_t> wlist[kMaxL];
  int32_t max_copies[kMaxL] = {};   // max #written positions per index
  Affine aff;

  // lazily uploaded device copies, per device ordinal
  struct DevCopy { int dev = -1; void *blob = nullptr; SepDev sep{}; LayoutDesc *desc = nullptr; };
  std::mutex mu;
  std::vector<DevCopy> dev;

  ~Layout();
};

// host-side compile; returns status and a thread-local error via set_error
alt_status compile_layout(int32_t lrank, const int64_t *lshape, const alt_prim *prims,
                          int32_t np, Layout *L);

// host G (phys coords -> logical; returns false for a structural zero) and
// F (logical -> owner phys coords; false if no copy)
bool host_G(const LayoutDesc &D, const int64_t *phys, int64_t *logical);
bool host_F(const LayoutDesc &D, const int64_t *logical, int64_t *phys);

// upload (once per device) and return device pointers
alt_status device_tables(Layout *L, SepDev *sep, const LayoutDesc **desc);

void set_error(const char *fmt, ...);

}  // namespace alt

struct alt_layout_s {
  alt::Layout impl;
};
