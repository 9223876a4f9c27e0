/*
 * alt_oracle.c — fp64 CPU ORACLE for ALT's hot path.  TEST INFRASTRUCTURE.
 *
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline leg /
 * `--impl reference` arm may load this library.  It shares no code, header,
 * table or constant with the product (paper_conf_eurosys_xuxpwwwdxcwc23_b200/
 * and include/): primitives are passed in as plain int arrays and every map
 * is re-derived here from the paper text.
 *
 * Paper: Xu et al., ALT, EuroSys '23.  "P:a-b" = PAPER.md lines a-b.
 *
 *   O1  layout semantics: split / reorder / fuse (Table 1),
 *       unfold (§4.1.2), pad; primitives applied in
 *       sequence order.  G = physical -> logical (or "structural
 *       zero"), F = logical -> canonical (owner) physical.
 *   O2  materialise / relayout (conversion operator, Fig. 5a)
 *   O3  direct conv2d, textbook definition (P:498-514 computes this sum)
 *   O4  layout-native conv through Eq. (1) on the unfolded input
 *       of Fig. 2 / Fig. 3
 *   O5  GEMM C = A B
 *   O6  epilogue act(scale*acc + bias + residual) (bias + ReLU, P:2475-2477;
 *       elementwise Y[i] = F(X[i]))
 *
 * Readings of silent / garbled passages are the DESIGN.md "Readings" table
 * (A1-A22).  Every function here is pinned by tests/test_oracle_*.py against
 * paper examples, library routines (numpy / torch float64) or brute force.
 *
 * Precision: all arithmetic in fp64; operands arrive as raw 16-bit (bf16) or
 * 32-bit (fp32) words and are converted exactly.
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#define OR_MAXR 12
#define OR_MAXP 16

/* ------------------------------------------------------------------ O1 --- */
typedef struct {
  int lrank;
  int np;
  int kind[OR_MAXP], dim[OR_MAXP], n[OR_MAXP];
  long long v[OR_MAXP][10];
  int rank[OR_MAXP + 1];                /* rank after s primitives          */
  long long shp[OR_MAXP + 1][OR_MAXR];  /* shape after s primitives         */
} orc_layout;

enum { K_SPLIT = 0, K_REORDER = 1, K_FUSE = 2, K_UNFOLD = 3, K_PAD = 4 };
enum { E_OK = 0, E_INVALID = 1, E_SHAPE = 2, E_NONDIV = 3, E_LOSSY = 4 };

static long long ceil_div(long long a, long long b) { return (a + b - 1) / b; }

/* Build the per-stage shapes.  Returns an E_* code. */
int orc_layout_build(int lrank, const long long *lshape, int np,
                     const int *kind, const int *dim, const int *n,
                     const long long *v /* np x 10 */, orc_layout *L) {
  memset(L, 0, sizeof(*L));
  if (lrank < 1 || lrank > 8 || np < 0 || np > OR_MAXP) return E_INVALID;
  L->lrank = lrank;
  L->np = np;
  L->rank[0] = lrank;
  for (int d = 0; d < lrank; d++) {
    if (lshape[d] < 1) return E_INVALID;
    L->shp[0][d] = lshape[d];
  }
  for (int s = 0; s < np; s++) {
    L->kind[s] = kind[s];
    L->dim[s] = dim[s];
    L->n[s] = n[s];
    for (int q = 0; q < 10; q++) L->v[s][q] = v[s * 10 + q];
    int r = L->rank[s];
    const long long *D = L->shp[s];
    long long *E = L->shp[s + 1];
    int k = dim[s];
    switch (kind[s]) {
      case K_SPLIT: {  /* Table 1: N_k -> F_1 .. F_m */
        int m = n[s];
        if (k < 0 || k >= r || m < 1 || r - 1 + m > OR_MAXR) return E_INVALID;
        long long prod = 1;
        for (int l = 0; l < m; l++) {
          if (L->v[s][l] < 1) return E_INVALID;
          prod *= L->v[s][l];
        }
        if (prod != D[k]) return E_NONDIV;
        int o = 0;
        for (int d = 0; d < k; d++) E[o++] = D[d];
        for (int l = 0; l < m; l++) E[o++] = L->v[s][l];
        for (int d = k + 1; d < r; d++) E[o++] = D[d];
        L->rank[s + 1] = o;
        break;
      }
      case K_REORDER: {  /* Table 1: N_p(1) .. N_p(n) */
        if (n[s] != r) return E_INVALID;
        int seen[OR_MAXR] = {0};
        for (int j = 0; j < r; j++) {
          long long p = L->v[s][j];
          if (p < 0 || p >= r || seen[p]) return E_INVALID;
          seen[p] = 1;
          E[j] = D[p];
        }
        L->rank[s + 1] = r;
        break;
      }
      case K_FUSE: {  /* Table 1: consecutive dims k..k+m-1 -> one dim */
        int m = n[s];
        if (k < 0 || m < 2 || k + m > r) return E_INVALID;
        int o = 0;
        for (int d = 0; d < k; d++) E[o++] = D[d];
        long long prod = 1;
        for (int l = 0; l < m; l++) prod *= D[k + l];
        E[o++] = prod;
        for (int d = k + m; d < r; d++) E[o++] = D[d];
        L->rank[s + 1] = o;
        break;
      }
      case K_UNFOLD: {  /* §4.1.2: D -> (ceil((D-B)/S)+1, B) */
        long long B = L->v[s][0], S = L->v[s][1];
        if (k < 0 || k >= r || r + 1 > OR_MAXR || S < 1) return E_INVALID;
        if (B < 1 || B > D[k]) return E_SHAPE;
        int o = 0;
        for (int d = 0; d < k; d++) E[o++] = D[d];
        E[o++] = ceil_div(D[k] - B, S) + 1;
        E[o++] = B;
        for (int d = k + 1; d < r; d++) E[o++] = D[d];
        L->rank[s + 1] = o;
        break;
      }
      case K_PAD: {  /* append lo / hi zeros on one dim */
        long long lo = L->v[s][0], hi = L->v[s][1];
        if (k < 0 || k >= r || lo < 0 || hi < 0) return E_INVALID;
        for (int d = 0; d < r; d++) E[d] = D[d];
        E[k] = D[k] + lo + hi;
        L->rank[s + 1] = r;
        break;
      }
      default:
        return E_INVALID;
    }
    if (L->rank[s + 1] > OR_MAXR) return E_INVALID;
  }
  if (L->rank[np] > 10) return E_INVALID;
  return E_OK;
}

int orc_phys_rank(const orc_layout *L) { return L->rank[L->np]; }
void orc_phys_shape(const orc_layout *L, long long *out) {
  for (int d = 0; d < L->rank[L->np]; d++) out[d] = L->shp[L->np][d];
}
long long orc_phys_numel(const orc_layout *L) {
  long long t = 1;
  for (int d = 0; d < L->rank[L->np]; d++) t *= L->shp[L->np][d];
  return t;
}
long long orc_logical_numel(const orc_layout *L) {
  long long t = 1;
  for (int d = 0; d < L->lrank; d++) t *= L->shp[0][d];
  return t;
}

/* G: physical coordinates (after all primitives) -> logical coordinates.
 * Walks the primitives in reverse order, undoing one at a time.
 * Returns 1 if the position holds logical element `out`, 0 if it is a
 * structural zero (pad region or unfold overhang). */
int orc_G(const orc_layout *L, const long long *phys, long long *out) {
  long long cur[OR_MAXR], prev[OR_MAXR];
  int r = L->rank[L->np];
  for (int d = 0; d < r; d++) cur[d] = phys[d];
  for (int s = L->np - 1; s >= 0; s--) {
    const long long *D = L->shp[s];  /* shape before primitive s */
    int rp = L->rank[s];
    int k = L->dim[s];
    switch (L->kind[s]) {
      case K_SPLIT: {
        /* i_k = sum_l j_{k+l} * prod_{q>l} F_q  (inverse of Table 1 row) */
        int m = L->n[s];
        for (int d = 0; d < k; d++) prev[d] = cur[d];
        long long i = 0;
        for (int l = 0; l < m; l++) i = i * L->v[s][l] + cur[k + l];
        prev[k] = i;
        for (int d = k + 1; d < rp; d++) prev[d] = cur[d + m - 1];
        break;
      }
      case K_REORDER: {
        /* new dim j is old dim p(j): old index i_{p(j)} = j'_j */
        for (int j = 0; j < rp; j++) prev[L->v[s][j]] = cur[j];
        break;
      }
      case K_FUSE: {
        /* e = i_k N_{k+1..} + ... + i_{k+m-1}: recover the row-major digits */
        int m = L->n[s];
        for (int d = 0; d < k; d++) prev[d] = cur[d];
        long long e = cur[k];
        for (int l = m - 1; l >= 0; l--) {
          prev[k + l] = e % D[k + l];
          e /= D[k + l];
        }
        for (int d = k + m; d < rp; d++) prev[d] = cur[d - m + 1];
        break;
      }
      case K_UNFOLD: {
        /* tile t, offset b -> i = t*S + b; beyond the original extent the
         * overhanging last tile holds zeros (reading A3). */
        long long S = L->v[s][1];
        for (int d = 0; d < k; d++) prev[d] = cur[d];
        long long i = cur[k] * S + cur[k + 1];
        if (i >= D[k]) return 0;
        prev[k] = i;
        for (int d = k + 1; d < rp; d++) prev[d] = cur[d + 1];
        break;
      }
      case K_PAD: {
        long long lo = L->v[s][0];
        for (int d = 0; d < rp; d++) prev[d] = cur[d];
        long long i = cur[k] - lo;
        if (i < 0 || i >= D[k]) return 0;
        prev[k] = i;
        break;
      }
    }
    for (int d = 0; d < rp; d++) cur[d] = prev[d];
    r = rp;
  }
  for (int d = 0; d < L->lrank; d++) out[d] = cur[d];
  return 1;
}

/* F: logical coordinates -> canonical (owner) physical coordinates.
 * Applies the primitives in order (Table 1 "transformed accessing
 * expressions").  For unfold the owner tile is t = min(floor(i/S), T-1)
 * (reading A5).  Returns 1, or 0 if the element has no copy (B < S gap). */
int orc_F(const orc_layout *L, const long long *logical, long long *out) {
  long long cur[OR_MAXR], nxt[OR_MAXR];
  for (int d = 0; d < L->lrank; d++) cur[d] = logical[d];
  for (int s = 0; s < L->np; s++) {
    int r = L->rank[s];
    int k = L->dim[s];
    const long long *E = L->shp[s + 1];
    switch (L->kind[s]) {
      case K_SPLIT: {
        /* (i/F_{2..m}, ..., (i/F_m) mod F_{m-1}, i mod F_m) */
        int m = L->n[s];
        for (int d = 0; d < k; d++) nxt[d] = cur[d];
        long long i = cur[k];
        for (int l = m - 1; l >= 0; l--) {
          nxt[k + l] = i % L->v[s][l];
          i /= L->v[s][l];
        }
        for (int d = k + 1; d < r; d++) nxt[d + m - 1] = cur[d];
        break;
      }
      case K_REORDER: {
        for (int j = 0; j < r; j++) nxt[j] = cur[L->v[s][j]];
        break;
      }
      case K_FUSE: {
        int m = L->n[s];
        const long long *D = L->shp[s];
        for (int d = 0; d < k; d++) nxt[d] = cur[d];
        long long e = 0;
        for (int l = 0; l < m; l++) e = e * D[k + l] + cur[k + l];
        nxt[k] = e;
        for (int d = k + m; d < r; d++) nxt[d - m + 1] = cur[d];
        break;
      }
      case K_UNFOLD: {
        long long B = L->v[s][0], S = L->v[s][1];
        long long T = E[k];
        for (int d = 0; d < k; d++) nxt[d] = cur[d];
        long long i = cur[k];
        long long t = i / S;
        if (t > T - 1) t = T - 1;
        long long b = i - t * S;
        if (b >= B) return 0;
        nxt[k] = t;
        nxt[k + 1] = b;
        for (int d = k + 1; d < r; d++) nxt[d + 1] = cur[d];
        break;
      }
      case K_PAD: {
        for (int d = 0; d < r; d++) nxt[d] = cur[d];
        nxt[k] = cur[k] + L->v[s][0];
        break;
      }
    }
    for (int d = 0; d < L->rank[s + 1]; d++) cur[d] = nxt[d];
  }
  for (int d = 0; d < L->rank[L->np]; d++) out[d] = cur[d];
  return 1;
}

static long long linear(const long long *c, const long long *shape, int r) {
  long long j = 0;
  for (int d = 0; d < r; d++) j = j * shape[d] + c[d];
  return j;
}
static void unlinear(long long j, const long long *shape, int r, long long *c) {
  for (int d = r - 1; d >= 0; d--) {
    c[d] = j % shape[d];
    j /= shape[d];
  }
}

/* linear-index convenience wrappers used by the Python side */
int orc_G_linear(const orc_layout *L, long long j, long long *logical) {
  long long c[OR_MAXR];
  unlinear(j, L->shp[L->np], L->rank[L->np], c);
  return orc_G(L, c, logical);
}
long long orc_F_linear(const orc_layout *L, const long long *logical) {
  long long c[OR_MAXR];
  if (!orc_F(L, logical, c)) return -1;
  return linear(c, L->shp[L->np], L->rank[L->np]);
}

/* ------------------------------------------------------------------ O2 --- */
/* Word copies of width wb (2 or 4 bytes).  dst[j] = G(j) = zero ? 0 :
 * src[...].  Returns E_OK or E_LOSSY. */
static void put_word(void *p, long long j, int wb, uint32_t w) {
  if (wb == 2) ((uint16_t *)p)[j] = (uint16_t)w;
  else ((uint32_t *)p)[j] = w;
}
static uint32_t get_word(const void *p, long long j, int wb) {
  return wb == 2 ? ((const uint16_t *)p)[j] : ((const uint32_t *)p)[j];
}

/* P[j] = L[G(j)] (row-major logical tensor -> physical layout). */
int orc_materialize(const orc_layout *L, const void *logical, void *phys, int wb) {
  long long n = orc_phys_numel(L);
  int r = L->rank[L->np];
  int err = E_OK;
#pragma omp parallel for schedule(static)
  for (long long j = 0; j < n; j++) {
    long long c[OR_MAXR], l[OR_MAXR];
    unlinear(j, L->shp[L->np], r, c);
    if (orc_G(L, c, l)) put_word(phys, j, wb, get_word(logical, linear(l, L->shp[0], L->lrank), wb));
    else put_word(phys, j, wb, 0);
  }
  return err;
}

/* logical[i] = P[F(i)] (physical -> row-major logical). E_LOSSY if some
 * element has no copy. */
int orc_unmaterialize(const orc_layout *L, const void *phys, void *logical, int wb) {
  long long n = orc_logical_numel(L);
  int lossy = 0;
#pragma omp parallel for schedule(static) reduction(| : lossy)
  for (long long i = 0; i < n; i++) {
    long long l[OR_MAXR], c[OR_MAXR];
    unlinear(i, L->shp[0], L->lrank, l);
    if (!orc_F(L, l, c)) { lossy |= 1; put_word(logical, i, wb, 0); continue; }
    put_word(logical, i, wb, get_word(phys, linear(c, L->shp[L->np], L->rank[L->np]), wb));
  }
  return lossy ? E_LOSSY : E_OK;
}

/* Checks that a physical buffer is a consistent image of some logical
 * tensor: every structural-zero position holds word 0 and every copy of a
 * logical element equals its owner copy.  Returns the number of violating
 * positions (0 = consistent). */
long long orc_check_consistent(const orc_layout *L, const void *phys, int wb) {
  long long n = orc_phys_numel(L);
  int r = L->rank[L->np];
  long long bad = 0;
#pragma omp parallel for schedule(static) reduction(+ : bad)
  for (long long j = 0; j < n; j++) {
    long long c[OR_MAXR], l[OR_MAXR], o[OR_MAXR];
    unlinear(j, L->shp[L->np], r, c);
    uint32_t w = get_word(phys, j, wb);
    if (!orc_G(L, c, l)) { bad += (w != 0); continue; }
    if (!orc_F(L, l, o)) { bad += 1; continue; }
    bad += (w != get_word(phys, linear(o, L->shp[L->np], r), wb));
  }
  return bad;
}

/* Conversion operator (Fig. 5a): dst[j] = G_dst(j) zero ? 0 :
 * src[F_src(G_dst(j))].  Logical shapes must agree. */
int orc_relayout(const orc_layout *S, const void *src, const orc_layout *D, void *dst, int wb) {
  if (S->lrank != D->lrank) return E_SHAPE;
  for (int d = 0; d < S->lrank; d++)
    if (S->shp[0][d] != D->shp[0][d]) return E_SHAPE;
  long long n = orc_phys_numel(D);
  int r = D->rank[D->np];
  int lossy = 0;
#pragma omp parallel for schedule(static) reduction(| : lossy)
  for (long long j = 0; j < n; j++) {
    long long c[OR_MAXR], l[OR_MAXR], sc[OR_MAXR];
    unlinear(j, D->shp[D->np], r, c);
    if (!orc_G(D, c, l)) { put_word(dst, j, wb, 0); continue; }
    if (!orc_F(S, l, sc)) { lossy |= 1; put_word(dst, j, wb, 0); continue; }
    put_word(dst, j, wb, get_word(src, linear(sc, S->shp[S->np], S->rank[S->np]), wb));
  }
  return lossy ? E_LOSSY : E_OK;
}

/* ---------------------------------------------------------- word -> fp64 */
static double word_to_f64(uint32_t w, int wb) {
  union { uint32_t u; float f; } cv;
  cv.u = (wb == 2) ? (w << 16) : w;  /* bf16 is the top half of an fp32 */
  return (double)cv.f;
}

/* Read a whole operand through its layout into a row-major fp64 logical
 * array (F map + exact conversion).  E_LOSSY if an element has no copy. */
int orc_read_logical(const orc_layout *L, const void *phys, int wb, double *out) {
  long long n = orc_logical_numel(L);
  int lossy = 0;
#pragma omp parallel for schedule(static) reduction(| : lossy)
  for (long long i = 0; i < n; i++) {
    long long l[OR_MAXR], c[OR_MAXR];
    unlinear(i, L->shp[0], L->lrank, l);
    if (!orc_F(L, l, c)) { lossy |= 1; out[i] = 0.0; continue; }
    out[i] = word_to_f64(get_word(phys, linear(c, L->shp[L->np], L->rank[L->np]), wb), wb);
  }
  return lossy ? E_LOSSY : E_OK;
}

/* present[i] = 1 when logical element i has a copy in the layout (F defined) */
void orc_present_mask(const orc_layout *L, unsigned char *present) {
  long long n = orc_logical_numel(L);
#pragma omp parallel for schedule(static)
  for (long long i = 0; i < n; i++) {
    long long l[OR_MAXR], c[OR_MAXR];
    unlinear(i, L->shp[0], L->lrank, l);
    present[i] = (unsigned char)(orc_F(L, l, c) ? 1 : 0);
  }
}

/* ------------------------------------------------------------------ O6 --- */
/* y = act(scale*acc + bias + residual); act 0 none, 1 ReLU, 2 ReLU6. */
static double epilogue(double acc, const double *scale, const double *bias,
                       const double *res, long long k, long long idx, int act) {
  double y = acc;
  if (scale) y = scale[k] * y;
  if (bias) y = y + bias[k];
  if (res) y = y + res[idx];
  if (act == 1) y = y > 0.0 ? y : 0.0;
  if (act == 2) y = y > 0.0 ? (y < 6.0 ? y : 6.0) : 0.0;
  return y;
}

/* ------------------------------------------------------------------ O3 --- */
/* Direct (textbook) conv2d on fp64 row-major logical arrays:
 *   y[n,k,p,q] = sum_{c<C/g} sum_{r<R} sum_{s<S}
 *                x[n, g(k) C/g + c, p V_h - pad_h + d_h r, q V_w - pad_w + d_w s] w[k,c,r,s]
 * x = 0 outside [0,H) x [0,W); g(k) = floor(k groups / K); dilation d (DIL,
 * the paper's single-operator set P:1546-1549; d = 1 is plain C2D);
 * Ho = floor((H + 2 pad_h - d_h (R - 1) - 1) / V_h) + 1.  The sum runs in
 * (c, r, s) ascending order.  Images n0 <= n < n1 are computed (the rest of
 * y is left untouched).  p[] = {N,C,H,W,K,R,S,Vh,Vw,ph,pw,groups,dh,dw}. */
void orc_conv2d_f64(const long long *p, const double *x, const double *w,
                    const double *scale, const double *bias, const double *res,
                    int act, long long n0, long long n1, double *y) {
  long long N = p[0], C = p[1], H = p[2], W = p[3], K = p[4], R = p[5], S = p[6];
  long long Vh = p[7], Vw = p[8], ph = p[9], pw = p[10], G = p[11], dh = p[12], dw = p[13];
  (void)N;
  long long Ho = (H + 2 * ph - dh * (R - 1) - 1) / Vh + 1, Wo = (W + 2 * pw - dw * (S - 1) - 1) / Vw + 1;
  long long Cg = C / G;
#pragma omp parallel for collapse(2) schedule(dynamic)
  for (long long n = n0; n < n1; n++)
    for (long long k = 0; k < K; k++) {
      long long g = k * G / K;
      for (long long oh = 0; oh < Ho; oh++)
        for (long long ow = 0; ow < Wo; ow++) {
          double acc = 0.0;
          for (long long c = 0; c < Cg; c++)
            for (long long r = 0; r < R; r++)
              for (long long s = 0; s < S; s++) {
                long long ih = oh * Vh - ph + dh * r, iw = ow * Vw - pw + dw * s;
                if (ih < 0 || ih >= H || iw < 0 || iw >= W) continue;
                acc += x[((n * C + g * Cg + c) * H + ih) * W + iw] *
                       w[((k * Cg + c) * R + r) * S + s];
              }
          long long idx = ((n * K + k) * Ho + oh) * Wo + ow;
          y[idx] = epilogue(acc, scale, bias, res, k, idx, act);
        }
    }
}

/* ----------------------------------------------------------------- O3b --- */
/* Direct (textbook) 3-D convolution, the paper's C3D operator (
 * "for other convolutions (e.g., 3-D case), the template is similar",
 * P:1146-1150): on fp64 row-major logical arrays x[N,C,D,H,W],
 * w[K,C/G,T,R,S], y[N,K,Do,Ho,Wo],
 *   y[n,k,od,oh,ow] = sum_{c<C/G, t<T, r<R, s<S}
 *       x[n, g(k) C/G + c, od Vd - pd + dd t, oh Vh - ph + dh r, ow Vw - pw + dw s]
 *       * w[k, c, t, r, s]      (x = 0 outside the tensor),
 * summed in (c, t, r, s) ascending order, then the O6 epilogue.
 * p[] = {N,C,D,H,W,K,T,R,S, Vd,Vh,Vw, pd,ph,pw, dd,dh,dw, G}. */
void orc_conv3d_f64(const long long *p, const double *x, const double *w,
                    const double *scale, const double *bias, const double *res,
                    int act, double *y) {
  long long N = p[0], C = p[1], D = p[2], H = p[3], W = p[4], K = p[5], T = p[6], R = p[7], S = p[8];
  long long Vd = p[9], Vh = p[10], Vw = p[11], pd = p[12], ph = p[13], pw = p[14];
  long long dd = p[15], dh = p[16], dw = p[17], G = p[18];
  long long Do = (D + 2 * pd - dd * (T - 1) - 1) / Vd + 1;
  long long Ho = (H + 2 * ph - dh * (R - 1) - 1) / Vh + 1, Wo = (W + 2 * pw - dw * (S - 1) - 1) / Vw + 1;
  long long Cg = C / G;
#pragma omp parallel for collapse(2) schedule(dynamic)
  for (long long n = 0; n < N; n++)
    for (long long k = 0; k < K; k++) {
      long long g = k * G / K;
      for (long long od = 0; od < Do; od++)
        for (long long oh = 0; oh < Ho; oh++)
          for (long long ow = 0; ow < Wo; ow++) {
            double acc = 0.0;
            for (long long c = 0; c < Cg; c++)
              for (long long t = 0; t < T; t++)
                for (long long r = 0; r < R; r++)
                  for (long long s = 0; s < S; s++) {
                    long long id = od * Vd - pd + dd * t, ih = oh * Vh - ph + dh * r, iw = ow * Vw - pw + dw * s;
                    if (id < 0 || id >= D || ih < 0 || ih >= H || iw < 0 || iw >= W) continue;
                    acc += x[(((n * C + g * Cg + c) * D + id) * H + ih) * W + iw] *
                           w[(((k * Cg + c) * T + t) * R + r) * S + s];
                  }
            long long idx = (((n * K + k) * Do + od) * Ho + oh) * Wo + ow;
            y[idx] = epilogue(acc, scale, bias, res, k, idx, act);
          }
    }
}

/* Same definition evaluated one output at a time, reading x and w through
 * their layouts' F maps directly (for sampled checks at full size).
 * pts: npts x 4 (n,k,p,q). */
int orc_conv2d_points(const long long *p, const orc_layout *XL, const void *x,
                      const orc_layout *WL, const void *w, int wb,
                      const double *scale, const double *bias,
                      const orc_layout *RL, const void *res, int act,
                      long long npts, const long long *pts, double *out) {
  long long C = p[1], H = p[2], W = p[3], K = p[4], R = p[5], S = p[6];
  long long Vh = p[7], Vw = p[8], ph = p[9], pw = p[10], G = p[11], dh = p[12], dw = p[13];
  long long Cg = C / G;
  int lossy = 0;
#pragma omp parallel for schedule(dynamic) reduction(| : lossy)
  for (long long t = 0; t < npts; t++) {
    long long n = pts[4 * t], k = pts[4 * t + 1], oh = pts[4 * t + 2], ow = pts[4 * t + 3];
    long long g = k * G / K;
    double acc = 0.0;
    long long li[OR_MAXR], pc[OR_MAXR];
    for (long long c = 0; c < Cg; c++)
      for (long long r = 0; r < R; r++)
        for (long long s = 0; s < S; s++) {
          long long ih = oh * Vh - ph + dh * r, iw = ow * Vw - pw + dw * s;
          if (ih < 0 || ih >= H || iw < 0 || iw >= W) continue;
          li[0] = n; li[1] = g * Cg + c; li[2] = ih; li[3] = iw;
          if (!orc_F(XL, li, pc)) { lossy = 1; continue; }
          double xv = word_to_f64(get_word(x, linear(pc, XL->shp[XL->np], XL->rank[XL->np]), wb), wb);
          li[0] = k; li[1] = c; li[2] = r; li[3] = s;
          if (!orc_F(WL, li, pc)) { lossy = 1; continue; }
          double wv = word_to_f64(get_word(w, linear(pc, WL->shp[WL->np], WL->rank[WL->np]), wb), wb);
          acc += xv * wv;
        }
    double y = acc;
    if (scale) y = scale[k] * y;
    if (bias) y = y + bias[k];
    if (res) {
      li[0] = n; li[1] = k; li[2] = oh; li[3] = ow;
      if (!orc_F(RL, li, pc)) lossy = 1;
      else y += word_to_f64(get_word(res, linear(pc, RL->shp[RL->np], RL->rank[RL->np]), wb), wb);
    }
    if (act == 1) y = y > 0.0 ? y : 0.0;
    if (act == 2) y = y > 0.0 ? (y < 6.0 ? y : 6.0) : 0.0;
    out[t] = y;
  }
  return lossy ? E_LOSSY : E_OK;
}

/* ------------------------------------------------------------------ O4 --- */
/* Layout-native conv of Fig. 3 on the overlapped-tiled input of Fig. 2.
 * xu is the physical fp64 buffer of layout
 *   NCHW -> pad(H,ph,ph) -> pad(W,pw,pw) -> unfold(H,Bh,Sh) -> unfold(W,Bw,Sw)
 * i.e. physical shape [N][C][Th][Bh][Tw][Bw] (no reorder), with
 * Sh = Vh*ht, Bh = Vh*(ht-1)+R (reading A6) and likewise along W.
 * Every access Inp[V*i + r] of the padded input is rewritten by Eq. (1):
 *   T[V i + r] -> T[ floor(i / w) ][ V i + r - S floor(i / w) ],
 *   w = floor((B - M) / V) + 1       (M = window size)
 * The sum order (c, r, s ascending) equals O3's, so the result is bit-exact
 * equal to O3 (invariant I3). */
void orc_conv2d_unfold_native(const long long *p, long long ht, long long wt,
                              const double *xu, const double *w, double *y) {
  long long N = p[0], C = p[1], H = p[2], W = p[3], K = p[4], R = p[5], S = p[6];
  long long Vh = p[7], Vw = p[8], ph = p[9], pw = p[10];
  long long Ho = (H + 2 * ph - R) / Vh + 1, Wo = (W + 2 * pw - S) / Vw + 1;
  long long Hp = H + 2 * ph, Wp = W + 2 * pw;
  long long Bh = Vh * (ht - 1) + R, Sh = Vh * ht, Bw = Vw * (wt - 1) + S, Sw = Vw * wt;
  long long Th = (Hp - Bh + Sh - 1) / Sh + 1, Tw = (Wp - Bw + Sw - 1) / Sw + 1;
  long long wh = (Bh - R) / Vh + 1, ww = (Bw - S) / Vw + 1;  /* Eq. (1) w */
  (void)N;
#pragma omp parallel for collapse(2) schedule(dynamic)
  for (long long n = 0; n < N; n++)
    for (long long k = 0; k < K; k++)
      for (long long oh = 0; oh < Ho; oh++)
        for (long long ow = 0; ow < Wo; ow++) {
          double acc = 0.0;
          long long th = oh / wh, tw = ow / ww;
          for (long long c = 0; c < C; c++)
            for (long long r = 0; r < R; r++)
              for (long long s = 0; s < S; s++) {
                long long bh = Vh * oh + r - Sh * th;  /* Eq. (1) inner index */
                long long bw = Vw * ow + s - Sw * tw;
                long long idx = ((((n * C + c) * Th + th) * Bh + bh) * Tw + tw) * Bw + bw;
                /* the padded input holds 0 where O3 skips a term; adding an
                 * exact 0*w leaves the running sum unchanged (up to the sign
                 * of a zero sum), so O4 == O3 */
                acc += xu[idx] * w[((k * C + c) * R + r) * S + s];
              }
          y[((n * K + k) * Ho + oh) * Wo + ow] = acc;
        }
}

/* ------------------------------------------------------------------ O5 --- */
/* C[m,n] = sum_k A[m,k] B[k,n], k ascending, fp64 row-major logical arrays;
 * epilogue per column n.  Rows m0 <= m < m1. */
void orc_gemm_f64(long long M, long long N, long long K, const double *A,
                  const double *B, const double *scale, const double *bias,
                  const double *res, int act, long long m0, long long m1,
                  double *Cout) {
  (void)M;
#pragma omp parallel for schedule(dynamic)
  for (long long m = m0; m < m1; m++)
    for (long long n = 0; n < N; n++) {
      double acc = 0.0;
      for (long long k = 0; k < K; k++) acc += A[m * K + k] * B[k * N + n];
      Cout[m * N + n] = epilogue(acc, scale, bias, res, n, m * N + n, act);
    }
}

/* sizeof for the Python wrapper */
long long orc_layout_sizeof(void) { return (long long)sizeof(orc_layout); }

/* ------------------------------------------------------------------ O9 --- */
/* 2-D pooling (support op of the ResNet chains; not one of the
 * paper's operators): y[n,c,p,q] = max (kind 0) or mean (kind 1) of
 * x[n, c, p V_h - pad_h + r, q V_w - pad_w + s] over the in-bounds taps of the
 * R x S window.  p[] = {N,C,H,W,R,S,Vh,Vw,ph,pw}. */
void orc_pool2d_f64(const long long *p, const double *x, int kind, double *y) {
  long long N = p[0], C = p[1], H = p[2], W = p[3], R = p[4], S = p[5];
  long long Vh = p[6], Vw = p[7], ph = p[8], pw = p[9];
  long long Ho = (H + 2 * ph - R) / Vh + 1, Wo = (W + 2 * pw - S) / Vw + 1;
#pragma omp parallel for collapse(2) schedule(static)
  for (long long n = 0; n < N; n++)
    for (long long c = 0; c < C; c++)
      for (long long oh = 0; oh < Ho; oh++)
        for (long long ow = 0; ow < Wo; ow++) {
          double acc = kind == 0 ? -INFINITY : 0.0;
          long long cnt = 0;
          for (long long r = 0; r < R; r++)
            for (long long s = 0; s < S; s++) {
              long long ih = oh * Vh - ph + r, iw = ow * Vw - pw + s;
              if (ih < 0 || ih >= H || iw < 0 || iw >= W) continue;
              double v = x[((n * C + c) * H + ih) * W + iw];
              if (kind == 0) acc = v > acc ? v : acc;
              else acc += v;
              cnt++;
            }
          if (kind == 1) acc = cnt ? acc / (double)cnt : 0.0;
          y[((n * C + c) * Ho + oh) * Wo + ow] = acc;
        }
}
