// layout.cpp — compile an ALT primitive sequence into a Layout (host only,
// apart from the lazy device upload of its tables).
//
// Primitive semantics: split / reorder / fuse = Table 1;
// unfold = §4.1.2 (overhang reads as zero, reading A3; owner tile
// min(floor(i/S), T-1), reading A5); pad = P:783-786 (pad(dim, lo, hi), A7).
#include "layout.h"

#include <cuda_runtime.h>

#include <atomic>
#include <cstdarg>
#include <cstdio>
#include <cstring>

namespace alt {

static thread_local char g_err[512] = "";

void set_error(const char *fmt, ...) {
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(g_err, sizeof(g_err), fmt, ap);
  va_end(ap);
}
const char *last_error() { return g_err; }

Layout::~Layout() {
  for (auto &d : dev) {
    if (d.blob) {
      int cur = -1;
      cudaGetDevice(&cur);
      cudaSetDevice(d.dev);
      cudaFree(d.blob);
      cudaSetDevice(cur);
    }
  }
}

// ------------------------------------------------------ interpreter (host) --
// Per-stage value of one dimension while walking G backwards.
struct GVal {
  int64_t raw;   // unclamped (affine) value
  int64_t cl;    // clamped into range (the "owner" of a structural zero)
  bool ok;       // holds a real element
};

// G with per-dimension validity: phys -> logical (raw, clamped, valid).
static void g_detail(const LayoutDesc &D, const int64_t *phys, GVal *out) {
  GVal cur[kStageRank], prev[kStageRank];
  int r = D.rank[D.np];
  for (int d = 0; d < r; d++) cur[d] = {phys[d], phys[d], true};
  for (int s = D.np - 1; s >= 0; s--) {
    const int64_t *E = D.shp[s];
    int rp = D.rank[s], k = D.dim[s];
    switch (D.kind[s]) {
      case ALT_SPLIT: {
        int m = D.n[s];
        for (int d = 0; d < k; d++) prev[d] = cur[d];
        GVal g{0, 0, true};
        for (int l = 0; l < m; l++) {
          g.raw = g.raw * D.v[s][l] + cur[k + l].raw;
          g.cl = g.cl * D.v[s][l] + cur[k + l].cl;
          g.ok = g.ok && cur[k + l].ok;
        }
        prev[k] = g;
        for (int d = k + 1; d < rp; d++) prev[d] = cur[d + m - 1];
        break;
      }
      case ALT_REORDER:
        for (int j = 0; j < rp; j++) prev[D.v[s][j]] = cur[j];
        break;
      case ALT_FUSE: {
        int m = D.n[s];
        for (int d = 0; d < k; d++) prev[d] = cur[d];
        int64_t e = cur[k].cl;
        for (int l = m - 1; l >= 0; l--) {
          int64_t dig = e % E[k + l];
          prev[k + l] = {dig, dig, cur[k].ok};
          e /= E[k + l];
        }
        for (int d = k + m; d < rp; d++) prev[d] = cur[d - m + 1];
        break;
      }
      case ALT_UNFOLD: {
        int64_t S = D.v[s][1];
        for (int d = 0; d < k; d++) prev[d] = cur[d];
        int64_t raw = cur[k].raw * S + cur[k + 1].raw;
        int64_t c = cur[k].cl * S + cur[k + 1].cl;
        bool ok = cur[k].ok && cur[k + 1].ok && c < E[k];
        prev[k] = {raw, c < E[k] ? c : E[k] - 1, ok};
        for (int d = k + 1; d < rp; d++) prev[d] = cur[d + 1];
        break;
      }
      case ALT_PAD: {
        int64_t lo = D.v[s][0];
        for (int d = 0; d < rp; d++) prev[d] = cur[d];
        int64_t c = cur[k].cl - lo;
        bool ok = cur[k].ok && c >= 0 && c < E[k];
        prev[k] = {cur[k].raw - lo, c < 0 ? 0 : (c >= E[k] ? E[k] - 1 : c), ok};
        break;
      }
    }
    for (int d = 0; d < rp; d++) cur[d] = prev[d];
    r = rp;
  }
  for (int d = 0; d < D.lrank; d++) out[d] = cur[d];
}

bool host_G(const LayoutDesc &D, const int64_t *phys, int64_t *logical) {
  GVal g[kStageRank];
  g_detail(D, phys, g);
  bool ok = true;
  for (int d = 0; d < D.lrank; d++) {
    logical[d] = g[d].cl;
    ok = ok && g[d].ok;
  }
  return ok;
}

bool host_F(const LayoutDesc &D, const int64_t *logical, int64_t *phys) {
  int64_t cur[kStageRank], nxt[kStageRank];
  for (int d = 0; d < D.lrank; d++) cur[d] = logical[d];
  for (int s = 0; s < D.np; s++) {
    int r = D.rank[s], k = D.dim[s];
    const int64_t *E = D.shp[s];
    const int64_t *E1 = D.shp[s + 1];
    switch (D.kind[s]) {
      case ALT_SPLIT: {
        int m = D.n[s];
        for (int d = 0; d < k; d++) nxt[d] = cur[d];
        int64_t i = cur[k];
        for (int l = m - 1; l >= 0; l--) {
          nxt[k + l] = i % D.v[s][l];
          i /= D.v[s][l];
        }
        for (int d = k + 1; d < r; d++) nxt[d + m - 1] = cur[d];
        break;
      }
      case ALT_REORDER:
        for (int j = 0; j < r; j++) nxt[j] = cur[D.v[s][j]];
        break;
      case ALT_FUSE: {
        int m = D.n[s];
        for (int d = 0; d < k; d++) nxt[d] = cur[d];
        int64_t e = 0;
        for (int l = 0; l < m; l++) e = e * E[k + l] + cur[k + l];
        nxt[k] = e;
        for (int d = k + m; d < r; d++) nxt[d - m + 1] = cur[d];
        break;
      }
      case ALT_UNFOLD: {
        int64_t B = D.v[s][0], S = D.v[s][1], T = E1[k];
        for (int d = 0; d < k; d++) nxt[d] = cur[d];
        int64_t t = cur[k] / S;
        if (t > T - 1) t = T - 1;
        int64_t b = cur[k] - t * S;
        if (b >= B) return false;
        nxt[k] = t;
        nxt[k + 1] = b;
        for (int d = k + 1; d < r; d++) nxt[d + 1] = cur[d];
        break;
      }
      case ALT_PAD:
        for (int d = 0; d < r; d++) nxt[d] = cur[d];
        nxt[k] = cur[k] + D.v[s][0];
        break;
    }
    for (int d = 0; d < D.rank[s + 1]; d++) cur[d] = nxt[d];
  }
  for (int d = 0; d < D.prank; d++) phys[d] = cur[d];
  return true;
}

// --------------------------------------------------------------- compile --
alt_status compile_layout(int32_t lrank, const int64_t *lshape, const alt_prim *prims,
                          int32_t np, Layout *L) {
  if (lrank < 1 || lrank > kMaxL || !lshape || np < 0 || np > ALT_MAX_PRIMS ||
      (np > 0 && !prims)) {
    set_error("alt_layout_create: bad rank %d / nprims %d", lrank, np);
    return ALT_E_INVALID;
  }
  static std::atomic<uint64_t> next_serial{1};
  L->serial = next_serial.fetch_add(1);
  LayoutDesc &D = L->desc;
  memset(&D, 0, sizeof(D));
  L->lrank = lrank;
  L->np = np;
  D.lrank = lrank;
  D.np = np;
  D.rank[0] = lrank;
  L->lnumel = 1;
  uint32_t mask[ALT_MAX_PRIMS + 1][kStageRank];
  for (int d = 0; d < lrank; d++) {
    if (lshape[d] < 1) {
      set_error("alt_layout_create: logical extent %lld < 1", (long long)lshape[d]);
      return ALT_E_INVALID;
    }
    L->lshape[d] = lshape[d];
    D.shp[0][d] = lshape[d];
    mask[0][d] = 1u << d;
    L->lnumel *= lshape[d];
  }
  bool lossless = true, has_pad = false, has_unfold = false;
  for (int s = 0; s < np; s++) {
    const alt_prim &p = prims[s];
    L->prims[s] = p;
    D.kind[s] = p.kind;
    D.dim[s] = p.dim;
    D.n[s] = p.n;
    for (int q = 0; q < 10; q++) D.v[s][q] = p.v[q];
    int r = D.rank[s], k = p.dim;
    const int64_t *E = D.shp[s];
    int64_t *E1 = D.shp[s + 1];
    const uint32_t *M = mask[s];
    uint32_t *M1 = mask[s + 1];
    int o = 0;
    switch (p.kind) {
      case ALT_SPLIT: {
        int m = p.n;
        if (k < 0 || k >= r || m < 1 || m > 10 || r - 1 + m > kStageRank) {
          set_error("split: bad dim %d / #factors %d at rank %d", k, m, r);
          return ALT_E_INVALID;
        }
        int64_t prod = 1;
        for (int l = 0; l < m; l++) {
          if (p.v[l] < 1) { set_error("split: factor < 1"); return ALT_E_INVALID; }
          prod *= p.v[l];
        }
        if (prod != E[k]) {
          set_error("split: factors multiply to %lld, extent is %lld (pad first)",
                    (long long)prod, (long long)E[k]);
          return ALT_E_NONDIVISIBLE;
        }
        for (int d = 0; d < k; d++) { E1[o] = E[d]; M1[o++] = M[d]; }
        for (int l = 0; l < m; l++) { E1[o] = p.v[l]; M1[o++] = M[k]; }
        for (int d = k + 1; d < r; d++) { E1[o] = E[d]; M1[o++] = M[d]; }
        break;
      }
      case ALT_REORDER: {
        if (p.n != r) { set_error("reorder: n=%d != rank %d", p.n, r); return ALT_E_INVALID; }
        bool seen[kStageRank] = {};
        for (int j = 0; j < r; j++) {
          int64_t q = p.v[j];
          if (q < 0 || q >= r || seen[q]) { set_error("reorder: not a permutation"); return ALT_E_INVALID; }
          seen[q] = true;
          E1[j] = E[q];
          M1[j] = M[q];
        }
        o = r;
        break;
      }
      case ALT_FUSE: {
        int m = p.n;
        if (k < 0 || m < 2 || k + m > r) { set_error("fuse: bad dims %d..+%d at rank %d", k, m, r); return ALT_E_INVALID; }
        for (int d = 0; d < k; d++) { E1[o] = E[d]; M1[o++] = M[d]; }
        int64_t prod = 1;
        uint32_t mm = 0;
        for (int l = 0; l < m; l++) { prod *= E[k + l]; mm |= M[k + l]; }
        E1[o] = prod;
        M1[o++] = mm;
        for (int d = k + m; d < r; d++) { E1[o] = E[d]; M1[o++] = M[d]; }
        break;
      }
      case ALT_UNFOLD: {
        int64_t B = p.v[0], S = p.v[1];
        if (k < 0 || k >= r || r + 1 > kStageRank || S < 1) { set_error("unfold: bad dim/stride"); return ALT_E_INVALID; }
        if (B < 1 || B > E[k]) { set_error("unfold: tile %lld outside [1, %lld]", (long long)B, (long long)E[k]); return ALT_E_SHAPE; }
        int64_t T = (E[k] - B + S - 1) / S + 1;
        if (B < S && B < E[k]) lossless = false;        // gaps (A4)
        if ((T - 1) * S + B > E[k]) has_pad = true;     // overhang (A3)
        if (T > 1 && B > S) has_unfold = true;          // duplicated elements
        for (int d = 0; d < k; d++) { E1[o] = E[d]; M1[o++] = M[d]; }
        E1[o] = T; M1[o++] = M[k];
        E1[o] = B; M1[o++] = M[k];
        for (int d = k + 1; d < r; d++) { E1[o] = E[d]; M1[o++] = M[d]; }
        break;
      }
      case ALT_PAD: {
        int64_t lo = p.v[0], hi = p.v[1];
        if (k < 0 || k >= r || lo < 0 || hi < 0) { set_error("pad: bad dim or negative amount"); return ALT_E_INVALID; }
        for (int d = 0; d < r; d++) { E1[d] = E[d]; M1[d] = M[d]; }
        E1[k] = E[k] + lo + hi;
        if (lo + hi > 0) has_pad = true;
        o = r;
        break;
      }
      default:
        set_error("unknown primitive kind %d", p.kind);
        return ALT_E_INVALID;
    }
    D.rank[s + 1] = o;
  }
  int pr = D.rank[np];
  if (pr > kMaxP) { set_error("physical rank %d > %d", pr, kMaxP); return ALT_E_INVALID; }
  L->prank = pr;
  D.prank = pr;
  L->pnumel = 1;
  for (int d = pr - 1; d >= 0; d--) {
    L->pshape[d] = D.shp[np][d];
    L->pstride[d] = L->pnumel;
    D.pstride[d] = L->pnumel;
    L->pnumel *= L->pshape[d];
  }
  L->flags = (lossless ? ALT_LOSSLESS : 0) | (has_pad ? ALT_HAS_PAD : 0) |
             (has_unfold ? ALT_HAS_UNFOLD : 0);

  // ---- separability and per-logical-dim tables
  bool sep = true;
  for (int p = 0; p < pr; p++) {
    uint32_t m = mask[np][p];
    if (m == 0 || (m & (m - 1))) sep = false;
  }
  L->separable = sep;
  if (!sep) return ALT_OK;
  L->flags |= ALT_SEPARABLE;
  for (int p = 0; p < pr; p++) L->pdim_owner[p] = __builtin_ctz(mask[np][p]);
  for (int d = 0; d < lrank; d++) {
    int64_t fp = 1;
    for (int p = pr - 1; p >= 0; p--)
      if (L->pdim_owner[p] == d) { L->pdim_rad[p] = (int32_t)fp; fp *= L->pshape[p]; }
    if (fp > (1ll << 30)) { set_error("layout footprint too large"); return ALT_E_INVALID; }
    L->footprint[d] = (int32_t)fp;
  }
  bool identity = !has_pad && !has_unfold && L->pnumel == L->lnumel;
  bool affine = true;
  int64_t phys[kMaxP], logical[kMaxL];
  for (int d = 0; d < lrank; d++) {
    const int64_t Dd = L->lshape[d];
    const int32_t fp = L->footprint[d];
    // owner offsets
    L->rd[d].assign(Dd, -1);
    for (int64_t i = 0; i < Dd; i++) {
      for (int q = 0; q < lrank; q++) logical[q] = 0;
      logical[d] = i;
      if (!host_F(D, logical, phys)) { L->flags &= ~ALT_LOSSLESS; continue; }
      int64_t off = 0;
      for (int p = 0; p < pr; p++)
        if (L->pdim_owner[p] == d) off += phys[p] * L->pstride[p];
      L->rd[d][i] = off;
    }
    // reverse table + write lists, raw affine check
    L->rev[d].assign(fp, 0);
    std::vector<int64_t> offs(fp);
    std::vector<int64_t> raw(fp);
    std::vector<int32_t> cnt(Dd + 1, 0);
    for (int32_t c = 0; c < fp; c++) {
      for (int p = 0; p < pr; p++) {
        phys[p] = (L->pdim_owner[p] == d) ? (c / L->pdim_rad[p]) % L->pshape[p] : 0;
      }
      GVal g[kStageRank];
      g_detail(D, phys, g);
      int64_t off = 0;
      for (int p = 0; p < pr; p++)
        if (L->pdim_owner[p] == d) off += phys[p] * L->pstride[p];
      offs[c] = off;
      raw[c] = g[d].raw;
      L->rev[d][c] = g[d].ok ? (int32_t)g[d].cl : -(int32_t)g[d].cl - 1;
      cnt[g[d].cl + 1]++;
    }
    L->wptr[d].assign(Dd + 1, 0);
    int32_t mx = 0;
    for (int64_t i = 0; i < Dd; i++) {
      L->wptr[d][i + 1] = L->wptr[d][i] + cnt[i + 1];
      mx = cnt[i + 1] > mx ? cnt[i + 1] : mx;
    }
    L->max_copies[d] = mx;
    L->wlist[d].assign(fp, 0);
    std::vector<int32_t> fill(L->wptr[d].begin(), L->wptr[d].end() - 1);
    for (int32_t c = 0; c < fp; c++) {
      int32_t v = L->rev[d][c];
      int64_t owner = v >= 0 ? v : -(int64_t)v - 1;
      L->wlist[d][fill[owner]++] = offs[c] * 2 + (v < 0 ? 1 : 0);
    }
    // affine descriptor: raw = sum coef_p j_p + off, valid <=> 0 <= raw < D
    int64_t off0 = raw[0];
    L->aff.off[d] = off0;
    for (int p = 0; p < pr; p++) {
      if (L->pdim_owner[p] != d) continue;
      L->aff.pd[p] = d;
      L->aff.coef[p] = L->pshape[p] > 1 ? raw[L->pdim_rad[p]] - off0 : 0;
    }
    for (int32_t c = 0; c < fp && affine; c++) {
      int64_t pred = off0;
      for (int p = 0; p < pr; p++)
        if (L->pdim_owner[p] == d) pred += ((c / L->pdim_rad[p]) % L->pshape[p]) * L->aff.coef[p];
      bool ok = L->rev[d][c] >= 0;
      if (pred != raw[c] || ok != (pred >= 0 && pred < Dd)) affine = false;
      if (ok && pred != L->rev[d][c]) affine = false;
    }
    // identity: row-major logical == physical
    int64_t rm = 1;
    for (int q = d + 1; q < lrank; q++) rm *= L->lshape[q];
    for (int64_t i = 0; i < Dd && identity; i++)
      if (L->rd[d][i] != i * rm) identity = false;
  }
  L->aff.ok = affine;
  if (identity) L->flags |= ALT_IDENTITY;
  return ALT_OK;
}

// ------------------------------------------------------------ device copy --
alt_status device_tables(Layout *L, SepDev *sep, const LayoutDesc **desc) {
  int dev = 0;
  if (cudaGetDevice(&dev) != cudaSuccess) { set_error("no CUDA device"); return ALT_E_CUDA; }
  std::lock_guard<std::mutex> g(L->mu);
  for (auto &d : L->dev) {
    if (d.dev == dev) {
      if (sep) *sep = d.sep;
      if (desc) *desc = d.desc;
      return ALT_OK;
    }
  }
  // blob: [desc][per d: rd | rev | wptr | wlist], 16-byte aligned pieces
  auto al = [](size_t x) { return (x + 15) & ~size_t(15); };
  size_t total = al(sizeof(LayoutDesc));
  if (L->separable) {
    for (int d = 0; d < L->lrank; d++) {
      total += al(L->rd[d].size() * 8) + al(L->rev[d].size() * 4) + al(L->wptr[d].size() * 4) +
               al(L->wlist[d].size() * 8);
    }
  }
  std::vector<uint8_t> host(total, 0);
  Layout::DevCopy dc;
  dc.dev = dev;
  if (cudaMalloc(&dc.blob, total) != cudaSuccess) {
    cudaGetLastError();
    set_error("cudaMalloc of layout tables failed");
    return ALT_E_NOMEM;
  }
  uint8_t *base = static_cast<uint8_t *>(dc.blob);
  size_t o = 0;
  memcpy(host.data(), &L->desc, sizeof(LayoutDesc));
  dc.desc = reinterpret_cast<LayoutDesc *>(base);
  o = al(sizeof(LayoutDesc));
  if (L->separable) {
    for (int d = 0; d < L->lrank; d++) {
      auto put = [&](const void *src, size_t bytes) {
        memcpy(host.data() + o, src, bytes);
        void *p = base + o;
        o += al(bytes);
        return p;
      };
      dc.sep.rd[d] = static_cast<const int64_t *>(put(L->rd[d].data(), L->rd[d].size() * 8));
      dc.sep.rev[d] = static_cast<const int32_t *>(put(L->rev[d].data(), L->rev[d].size() * 4));
      dc.sep.wptr[d] = static_cast<const int32_t *>(put(L->wptr[d].data(), L->wptr[d].size() * 4));
      dc.sep.wlist[d] = static_cast<const int64_t *>(put(L->wlist[d].data(), L->wlist[d].size() * 8));
    }
  }
  if (cudaMemcpy(dc.blob, host.data(), total, cudaMemcpyHostToDevice) != cudaSuccess) {
    cudaGetLastError();
    cudaFree(dc.blob);
    set_error("upload of layout tables failed");
    return ALT_E_CUDA;
  }
  L->dev.push_back(dc);
  if (sep) *sep = dc.sep;
  if (desc) *desc = dc.desc;
  return ALT_OK;
}

}  // namespace alt
