/*
 * alt.h — C-ABI of libalt.so: ALT's data-parallel hot path on B200 (sm_100a).
 *
 * Operators (conv2d, GEMM) executed directly on tensors stored in the tiled
 * layouts produced by ALT's layout primitives, plus the conversion kernels
 * between layouts.  Citations "P:a-b" are lines of the paper text
 * (Xu et al., "ALT: Breaking the Wall between Data Layout and Loop
 * Optimizations for Deep Learning Compilation", EuroSys '23) as extracted in
 * PAPER.md, followed by the section / table / equation they fall in.
 *
 * General conventions (apply to every call below)
 * -----------------------------------------------
 *  - Every call returns an alt_status.  Argument and layout validation happens
 *    synchronously before any launch; on failure nothing is launched and
 *    alt_last_error() (thread-local) holds a one-line detail.
 *  - Device buffers are allocated and owned by the caller.  The library never
 *    frees them.  Host pointers passed where a device pointer is expected are
 *    rejected with ALT_E_INVALID: there is NO CPU fallback.
 *  - alt_layout handles are allocated by alt_layout_create and released by
 *    alt_layout_destroy.  They are immutable after creation and may be shared
 *    across threads and streams.
 *  - alt_relayout / alt_conv2d / alt_matmul are asynchronous on `stream`
 *    (a cudaStream_t; NULL = legacy default stream).  Launch failures return
 *    ALT_E_CUDA; device faults surface at the caller's next synchronisation.
 *  - Dimensions are 0-based here (the paper numbers them from 1).
 */
#ifndef ALT_H_
#define ALT_H_

#include <stdint.h>
#include <stddef.h>

#ifdef __cplusplus
extern "C" {
#endif

/* forward declaration so this header does not need the CUDA headers */
typedef struct CUstream_st *alt_stream_t;

/* ---------------------------------------------------------------- status -- */
typedef enum {
  ALT_OK = 0,
  ALT_E_INVALID = 1,      /* bad argument: null, rank, unknown enum, host ptr  */
  ALT_E_SHAPE = 2,        /* layout logical shape != operand shape; B > D      */
  ALT_E_NONDIVISIBLE = 3, /* split factors do not multiply to the extent      */
  ALT_E_LOSSY = 4,        /* a needed element has no copy in the source layout */
  ALT_E_UNSUPPORTED = 5,  /* valid request without a kernel on the forced path */
  ALT_E_CUDA = 6,         /* CUDA runtime / driver error                      */
  ALT_E_NOMEM = 7         /* host or device allocation failed                 */
} alt_status;

const char *alt_status_str(alt_status s);
/* Thread-local detail of the last failing call on this thread ("" if none). */
const char *alt_last_error(void);

typedef enum { ALT_F32 = 0, ALT_BF16 = 1 } alt_dtype;

/* --------------------------------------------------------------- layouts -- */
/* Layout primitives, paper §4.1 (Table 1, Eq. 1
 * P:759-781).  A layout is the logical (row-major) tensor transformed by a
 * primitive sequence applied in order.
 *
 *   ALT_SPLIT   dim, n = #factors (>=1), v[0..n-1] = factors, outermost first.
 *               Requires prod(v) == extent(dim), else ALT_E_NONDIVISIBLE
 *               (non-divisible tiling is written as pad then split).
 *               Table 1 row "split".
 *   ALT_REORDER n = current rank, v = permutation: new dim j = old dim v[j].
 *               Table 1 row "reorder".
 *   ALT_FUSE    dim = first dim, n = number of consecutive dims (>=2);
 *               the fused index is row-major.  Table 1 row "fuse".
 *   ALT_UNFOLD  dim, v[0] = tile_size B, v[1] = stride S.
 *               Extent D becomes (T = ceil((D-B)/S)+1, B).  Requires
 *               1 <= B <= D and S >= 1, else ALT_E_SHAPE.  Positions with
 *               t*S+b >= D (overhang of the last tile) hold zero.  B < S
 *               leaves gaps: such a layout is LOSSY (no ALT_LOSSLESS flag).
 *   ALT_PAD     dim, v[0] = lo zeros, v[1] = hi zeros.
 */
#define ALT_MAX_RANK 10
#define ALT_MAX_PRIMS 16

typedef enum {
  ALT_SPLIT = 0, ALT_REORDER = 1, ALT_FUSE = 2, ALT_UNFOLD = 3, ALT_PAD = 4
} alt_prim_kind;

typedef struct {
  int32_t kind;               /* alt_prim_kind */
  int32_t dim;
  int32_t n;
  int32_t _pad;
  int64_t v[ALT_MAX_RANK];
} alt_prim;

typedef struct alt_layout_s *alt_layout;

/* Compile `prims` (nprims <= ALT_MAX_PRIMS) applied to a row-major logical
 * tensor of rank logical_rank (<= 8) and shape logical_shape into an
 * immutable layout.  Host only; no GPU needed.  Physical rank <= 10.
 * Errors: ALT_E_INVALID (bad dim/permutation/rank), ALT_E_NONDIVISIBLE,
 * ALT_E_SHAPE (unfold B > D or B < 1). */
alt_status alt_layout_create(int32_t logical_rank, const int64_t *logical_shape,
                             const alt_prim *prims, int32_t nprims,
                             alt_layout *out);
alt_status alt_layout_destroy(alt_layout l);

enum {
  ALT_LOSSLESS = 1,    /* every logical element has at least one copy      */
  ALT_HAS_PAD = 2,     /* some physical positions are structural zeros    */
  ALT_HAS_UNFOLD = 4,  /* some logical elements have >1 copy (or overhang) */
  ALT_SEPARABLE = 8,   /* each physical dim depends on one logical dim    */
  ALT_IDENTITY = 16    /* physical == logical row-major                    */
};

/* Physical shape (phys_shape has room for ALT_MAX_RANK entries), physical
 * element count and flags.  Any output pointer may be NULL. */
alt_status alt_layout_query(alt_layout l, int32_t *phys_rank,
                            int64_t *phys_shape, int64_t *phys_numel,
                            uint32_t *flags);
/* Logical rank and shape the layout was created for. */
alt_status alt_layout_logical(alt_layout l, int32_t *logical_rank,
                              int64_t *logical_shape);
/* Host-side evaluation of the compiled index maps (used by tests to check
 * the layout compiler against the oracle; never on the hot path).
 *  alt_layout_phys_to_logical: G(j) for the physical row-major linear index
 *    j; writes logical coordinates and returns *valid = 0 when j holds a
 *    structural zero (pad / unfold overhang), 1 otherwise.
 *  alt_layout_logical_to_phys: F(i) = canonical (owner) physical linear
 *    index of logical coordinates i; ALT_E_LOSSY if the element has no copy. */
alt_status alt_layout_phys_to_logical(alt_layout l, int64_t j,
                                      int64_t *logical_coords, int32_t *valid);
alt_status alt_layout_logical_to_phys(alt_layout l, const int64_t *logical_coords,
                                      int64_t *j);

/* ------------------------------------------------------- conversion op -- */
/* The runtime layout-conversion operator of Fig. 5a:
 *   dst[j] = G_dst(j) is a structural zero ? 0 : src[F_src(G_dst(j))]
 * for every physical position j of dst.  A bit copy (dtype only fixes the
 * element width: 4 B for ALT_F32, 2 B for ALT_BF16), so NaN payloads and -0
 * are preserved.  src_l and dst_l must have identical logical shapes
 * (ALT_E_SHAPE).  ALT_E_LOSSY if dst needs an element src has no copy of.
 * src and dst must not overlap. */
alt_status alt_relayout(alt_layout src_l, const void *src, alt_layout dst_l,
                        void *dst, alt_dtype dtype, alt_stream_t stream);

/* ------------------------------------------------ store_at / decouple_at -- */
/* The store_at primitive and its inverse ("fusing two tensors
 * together by attaching one to another ... attach each element of the bias
 * vector to each column of the weight matrix"; reading A26 in DESIGN.md):
 *   Z = store_at(A, b, dim):  Z has A's logical shape with extent E_dim + 1
 *   along dim; Z[i] = A[i] for i_dim < E_dim, Z[i] = b[i without dim] for
 *   i_dim == E_dim.
 * a is read through a_l (logical shape = A's), z written through z_l (logical
 * shape = A's with dim extended by one; every physical position, pad / unfold
 * overhang zeros included).  b is DENSE row-major over A's dims without dim
 * (prod of those extents elements).  All pointers device, caller-owned; a bit
 * copy of dtype-width elements (NaN payloads, -0 preserved).  Errors:
 * ALT_E_INVALID (NULL / host pointer, dim out of range, bad dtype),
 * ALT_E_SHAPE (z_l / a_l logical shapes inconsistent), ALT_E_LOSSY (a_l has
 * no copy of an element), ALT_E_CUDA (launch failure). */
alt_status alt_store_at(alt_layout a_l, const void *a, const void *b, int32_t dim,
                        alt_layout z_l, void *z, alt_dtype dtype, alt_stream_t stream);
/* (A, b) = decouple_at(Z, dim): the inverse; a written through a_l (all
 * physical positions), b dense row-major.  Same errors as alt_store_at. */
alt_status alt_decouple_at(alt_layout z_l, const void *z, int32_t dim, alt_layout a_l,
                           void *a, void *b, alt_dtype dtype, alt_stream_t stream);

/* ---------------------------------------------- operators on layouts -- */
/* conv2d, P:498-514 (Fig. 3): logical x [N,C,H,W],
 * w [K, C/groups, R, S], y [N, K, Ho, Wo], Ho = (H + 2 pad_h - R)/stride_h + 1
 *   y[n,k,p,q] = sum_{c,r,s} x[n, g(k)*C/groups + c, p*V_h - pad_h + r,
 *                               q*V_w - pad_w + s] * w[k,c,r,s]
 * with x = 0 outside [0,H)x[0,W) (semantic zero padding; if x_l itself holds
 * pad zeros the kernel may read them instead — identical results).
 * groups in {1, C (depthwise, K == C)}; other groups run on the generic
 * path; dil_h / dil_w > 1 (dilated conv, the paper's DIL operator): tap
 * (r, s) reads x[p V - pad + dil_h r, q V - pad + dil_w s], Ho = (H + 2 pad -
 * dil (R - 1) - 1) / V + 1; served by the tensor-core path (the tap offset
 * d r enters the TMA box coordinates) or the SIMT path (ALT_E_UNSUPPORTED when
 * the depthwise path is forced). */
typedef struct {
  int64_t N, C, H, W, K, R, S;
  int32_t stride_h, stride_w, pad_h, pad_w, dil_h, dil_w, groups;
  int32_t _pad;
} alt_conv2d_params;

typedef enum { ALT_ACT_NONE = 0, ALT_ACT_RELU = 1, ALT_ACT_RELU6 = 2 } alt_act;

/* Fused epilogue (the producer-side half of layout propagation, Fig. 5b,
 * P:870-879, and the elementwise ops of Figs. 6-7):
 *   y = act(scale[k] * acc + bias[k] + residual)
 * computed in fp32 and rounded once (RNE) to the output dtype, then stored
 * through y's layout: every unfold copy is written, pad positions get 0.
 * scale / bias are device fp32 arrays of length K (NULL = 1 / 0).
 * residual has y's logical shape, y's dtype, and its own layout.
 * flags & ALT_EPI_PADS_ZERO: the caller guarantees that y's pad / overhang
 * positions already hold 0 (e.g. a zero-initialised buffer only ever
 * written through this layout, as in a layer chain); the kernel then stores
 * the element positions only — a padded output layout is written by the
 * TMA-store epilogue instead of the per-element writer.  Unfold copies are
 * always all written. */
enum { ALT_EPI_PADS_ZERO = 1 };
typedef struct {
  const float *scale;
  const float *bias;
  const void *residual;
  alt_layout residual_l;
  int32_t act;                /* alt_act */
  int32_t flags;              /* ALT_EPI_* */
} alt_epilogue;

typedef enum {
  ALT_PATH_AUTO = 0,   /* tensor-core path when the layouts allow, else SIMT */
  ALT_PATH_TC = 1,     /* tcgen05 + TMA (ALT_E_UNSUPPORTED if not possible) */
  ALT_PATH_SIMT = 2,   /* generic CUDA-core gather through the index maps   */
  ALT_PATH_DW = 3      /* depthwise CUDA-core kernel (groups == C == K)     */
} alt_path;

/* Kernel ("loop") configuration; zeros mean "choose". For conv the M tile
 * is a (tile_n x tile_h x tile_w) block of output pixels with
 * tile_n*tile_h*tile_w == block_m. */
typedef struct {
  int32_t path;        /* alt_path */
  int32_t block_m;     /* 128 (or 256 with cta_pair) */
  int32_t block_n;     /* 32..256, multiple of 16 */
  int32_t block_k;     /* 64 (reduction slab per stage); tensor-core stride-1 3x3:
                          1 = request the halo mode (one A load per filter row,
                          the 3 taps along W read it shifted), 2 = refuse it;
                          reported back as 1 when the plan uses it */
  int32_t stages;      /* smem pipeline depth */
  int32_t cta_pair;    /* 0 auto, 1 = tcgen05 cta_group::2 CTA pair, 2 = one CTA */
  int32_t tile_n, tile_h, tile_w;
  int32_t split_k;     /* tensor-core path: 0 auto, 1 none, s = the reduction
                          is cut into s ranges whose fp32 partial tiles are
                          summed in split order by the last CTA to finish
                          (deterministic); for grids smaller than the GPU */
  int32_t split_cluster; /* 2: "tail split" — whole waves of output tiles run
                          unsplit and only the tiles of the last, partial wave
                          are split split_k ways (workspace form); removes
                          most of the wave-quantisation loss.
                          1: the split_k (2 or 4) ranges of a tile run as one
                          thread-block cluster and are summed in split order
                          through distributed shared memory, each CTA
                          finishing 1/split of the tile's rows (no workspace;
                          one CTA per tile part, block_n 128 / 256, no
                          residual, a TMA-store output layout; otherwise
                          ALT_E_UNSUPPORTED) */
} alt_kernel_cfg;

alt_status alt_conv2d(const alt_conv2d_params *p, alt_layout x_l, const void *x,
                      alt_layout w_l, const void *w, alt_layout y_l, void *y,
                      alt_dtype dtype, const alt_epilogue *epi /*nullable*/,
                      const alt_kernel_cfg *cfg /*nullable*/,
                      alt_stream_t stream);

/* 3-D convolution, the paper's C3D operator (its layout
 * template is "similar" to C2D's):
 *   y[n,k,od,oh,ow] = act(scale[k] * sum_{c<C/G, t<T, r<R, s<S}
 *       x[n, g(k) C/G + c, od Vd - pd + dd t, oh Vh - ph + dh r, ow Vw - pw + dw s]
 *       * w[k,c,t,r,s] + bias[k] + residual[n,k,od,oh,ow])
 * with x = 0 outside the tensor; Do = (D + 2 pd - dd (T - 1) - 1) / Vd + 1
 * (Ho, Wo alike).  Logical shapes: x [N,C,D,H,W], w [K,C/groups,T,R,S],
 * y / residual [N,K,Do,Ho,Wo], each in its own declared layout (errors,
 * ownership, asynchrony as alt_conv2d).  Tensor-core path: groups = 1, bf16 /
 * fp32 operands whose layouts admit a TMA view (channel tile innermost, the
 * depth dim plain or padded), output stored by TMA (no unfold copies; pads
 * only under ALT_EPI_PADS_ZERO), no residual; one output depth slice per
 * M tile (tile_n = 1).  Everything else: the generic CUDA-core path. */
typedef struct {
  int64_t N, C, D, H, W, K, T, R, S;
  int32_t stride_d, stride_h, stride_w, pad_d, pad_h, pad_w;
  int32_t dil_d, dil_h, dil_w, groups;
} alt_conv3d_params;
alt_status alt_conv3d(const alt_conv3d_params *p, alt_layout x_l, const void *x,
                      alt_layout w_l, const void *w, alt_layout y_l, void *y,
                      alt_dtype dtype, const alt_epilogue *epi /*nullable*/,
                      const alt_kernel_cfg *cfg /*nullable*/,
                      alt_stream_t stream);

/* GEMM: C[m,n] = sum_k A[m,k] B[k,n] with logical
 * A [M,K], B [K,N], C [M,N] in arbitrary declared layouts; epilogue as above
 * (per-column scale / bias, i.e. indexed by n). */
alt_status alt_matmul(int64_t M, int64_t N, int64_t K, alt_layout a_l,
                      const void *a, alt_layout b_l, const void *b,
                      alt_layout c_l, void *c, alt_dtype dtype,
                      const alt_epilogue *epi, const alt_kernel_cfg *cfg,
                      alt_stream_t stream);

/* GEMM consuming a store_at weight: z_l has logical shape
 * [K + 1, N] = store_at(B, bias, 0), i.e. column n is (B[:, n], bias[n]):
 *   C[m,n] = act(scale[n] * sum_{k<K} A[m,k] Z[k,n] + Z[K,n] + residual).
 * The contraction reads rows k < K of Z through z_l (the same kernels as
 * alt_matmul); the attached row Z[K, :] is the bias.  Separable z_l: the
 * epilogue reads bias[n] in place at Z's owner offset rd0[K] + rd1[n] (no
 * extra launch).  Non-separable z_l: the row is first gathered to fp32 by
 * one N-element launch on `stream` into stream-ordered scratch.  z_l must
 * be lossless (every element stored; else ALT_E_LOSSY).  epi may carry
 * scale / residual / act; epi->bias must be NULL (ALT_E_INVALID).  Other
 * errors as alt_matmul. */
alt_status alt_matmul_store_at(int64_t M, int64_t N, int64_t K, alt_layout a_l,
                               const void *a, alt_layout z_l, const void *z,
                               alt_layout c_l, void *c, alt_dtype dtype,
                               const alt_epilogue *epi, const alt_kernel_cfg *cfg,
                               alt_stream_t stream);

/* 2-D pooling on declared layouts (support op of the ResNet chains; not one
 * of the paper's operators).  Uses p's N, C, H, W, R, S (window),
 * stride and pad; K and groups are ignored.  x [N,C,H,W] -> y [N,C,Ho,Wo]:
 * kind 0 = max (padded taps skipped), 1 = average over in-bounds taps.
 * y is written through its layout (pad zeros, every unfold copy). */
typedef enum { ALT_POOL_MAX = 0, ALT_POOL_AVG = 1 } alt_pool_kind;
alt_status alt_pool2d(const alt_conv2d_params *p, alt_layout x_l, const void *x,
                      alt_layout y_l, void *y, alt_dtype dtype, int32_t kind,
                      alt_stream_t stream);

/* Describes which kernel the last alt_conv2d / alt_matmul on this thread
 * chose (alt_path) and its resolved cfg; for tests and the tuner. */
alt_status alt_last_plan(alt_kernel_cfg *cfg);

/* Number of kernels this library has launched in this process (all calls,
 * all streams); bench.py reports the difference across its timed region. */
uint64_t alt_launch_count(void);

/* ------------------------------------------- joint layout+loop tuning -- */
/* Bounded-grid replacement of ALT's joint tuning (§5): enumerate
 * layout template factors x kernel configs (P:1092-1179 templates), measure
 * each point on the device with CUDA events (L2 flushed between reps), and
 * return the fastest.  Synchronises `stream`.  Scratch is allocated and
 * freed inside.
 *
 * Conv template: x = N C/it H W it (it = x tile) with
 * optional pad(H,p,p)+pad(W,p,p) materialised, or the paper's overlapped
 * spatial tiles N H/ht W/wt C/it (ht+KH-1)(wt+KW-1) it (pad + unfold, Eq. 1;
 * stride V: B = V(ht-1)+KH, S = V ht, reading A6) when ht / wt are given;
 * w = K/ot' C/it' R S ot' it' (c innermost: K-major B, A11) or the paper's
 * O/ot' I/it' KH KW it' ot' (o innermost: MN-major B); y = N K/ot Ho Wo ot,
 * or N Ho/ht Wo/wt K/ot ht wt ot when ht | Ho and wt | Wo.
 * GEMM template: A = M/mt K/kt mt kt, B = N/nt K/kt nt kt
 * (K innermost) or the paper's K/kt N/nt kt nt (N innermost, MN-major),
 * C = M/mt N/nt mt nt.
 * Every grid point is timed as the median of `reps` L2-flushed launches;
 * the `topk` fastest are then re-measured (median of 3 x reps) and the best
 * re-measured point is returned.
 */
typedef enum { ALT_OP_CONV2D = 0, ALT_OP_MATMUL = 1 } alt_op_kind;

typedef struct { int64_t M, N, K; } alt_matmul_params;

#define ALT_TUNE_MAX_VALS 8
#define ALT_TUNE_NPARAMS 16
typedef struct {
  /* candidate values per template parameter; nvals[i] == 0 = default set.
   * conv:  0 it (x channel tile; the w c tile it' = it), 1 ot (y channel
   *        tile), 2 split_k (negative: -s = split_cluster form with s ranges),
   *        3 cta_pair (0 auto, 1 pair = BLOCK_M 256, 2 single CTA = 128),
   *        4 tile_h, 5 tile_w (kernel output-pixel tile), 6 block_n (the w k
   *        tile ot' = min(block_n, K)), 7 pad_x (0/1: materialise the conv
   *        zero padding in x), 8 ht, 9 wt (layout spatial tiles; 0 = none),
   *        10 stages (smem ring depth; 0 = deepest), 11 w order (0 c
   *        innermost, 1 the paper's it' ot'), 12 h't, 13 w't, 14 o't: the
   *        two-level output template N H/(h't ht) W/(w't wt) K/(o't ot)
   *        h't w't o't ht wt ot (0 or 1 = one level),
   *        15 halo (1: stride-1 3x3 taps along W from one row-shifted A
   *        load, cfg.block_k = 1; needs a pixel tile with tile_w >= Wo + 2)
   * gemm:  0 mt, 1 kt, 2 nt, 6 block_n, 10 stages, 11 B order (0 N/nt K/kt
   *        nt kt, 1 K/kt N/nt kt nt) */
  int64_t vals[ALT_TUNE_NPARAMS][ALT_TUNE_MAX_VALS];
  int32_t nvals[ALT_TUNE_NPARAMS];
  int32_t max_points;   /* budget: maximum measured points (<= 4096) */
  int32_t warmup, reps; /* per point */
  int32_t fix_x;        /* 1: keep x layout = fixed_x (propagated from a producer) */
  alt_layout fixed_x;
  int32_t topk;         /* re-measured finalists (0 = 3) */
} alt_tune_space;

typedef struct {
  alt_prim prims[3][ALT_MAX_PRIMS];   /* x/A, w/B, y/C primitive sequences */
  int32_t nprims[3];
  alt_kernel_cfg cfg;
  float best_us;
  int32_t measured;
} alt_tune_result;

alt_status alt_tune(alt_op_kind op, const void *op_params, alt_dtype dtype,
                    const alt_tune_space *space, alt_stream_t stream,
                    alt_tune_result *out, float *all_us /*nullable*/);

/* -------------------------------------------------- layout propagation -- */
/* Algorithm 1 plus the multi-producer rule over a
 * DAG of operators.  Host only.
 *  op_kind[i]: 0 = complex (conv/GEMM), 1 = elementwise (Y[i] = F(X[i])),
 *              2 = other simple op (pool, pad: a conversion boundary).
 *  Edge e carries tensor e from producer edge_src[e] (-1 = graph input) to
 *  consumer edge_dst[e] (-1 = graph output); edge_numel[e] = its element
 *  count (shape proxy for Alg. 1 line 10).  edge_in_idx[e] = input slot of
 *  the tensor at its consumer (0 = first input).
 *  edge_layout[e] = the tuned layout of e (output of a complex op, chosen by
 *  alt_tune) or NULL.  An IDENTITY layout is the empty sequence (A21).
 * Outputs per edge: src_edge[e] = the tuned edge whose layout e carries
 *  (-1 = none / default layout); conversion[e] = 1 if Alg. 1 inserts a
 *  conversion op on e (complex -> complex edge).  In this library the
 *  conversion is then fused into the producer's epilogue (it writes the
 *  consumer's layout directly), so no standalone conversion runs. */
alt_status alt_plan_chain(int32_t n_ops, const int32_t *op_kind, int32_t n_edges,
                          const int32_t *edge_src, const int32_t *edge_dst,
                          const int32_t *edge_in_idx, const int64_t *edge_numel,
                          const alt_layout *edge_layout, int32_t *src_edge,
                          int32_t *conversion);

#ifdef __cplusplus
}
#endif
#endif /* ALT_H_ */
