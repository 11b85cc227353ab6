// kernels_simt.cu -- fp32 CUDA-core (FFMA) path, MUCU_MATH_F32.
//
// Every convolution operation of every algorithm is expressed as a GEMM-shaped
// contraction  C[i][j] = alpha * sum_kk A(i,kk) * B(j,kk) + beta * C[i][j]
// whose operands are *views*: a dense matrix, the implicit im2col of x
// (FWD / WGRAD, Alg. 1 loop order n,k,h,w | c,s,r), or the implicit
// transposed-conv gather of dy (DGRAD).  One register-tiled SIMT kernel
// (128x128x8 block tile, 8x8 per thread, double-buffered shared memory) runs
// all of them; the fp32 path is FP32-ALU-bound (ridge ~11 flop/B), the
// tensor-core paths live in kernels_tc.cu.
//
// Determinism: the reduction over kk is one sequential loop per output
// element, so its order does not depend on the micro-batch size b (invariant I1
// of SURVEY 8(c)).  BackwardFilter splits the pixel reduction over
// CTAs and combines the partial tiles in split order through a per-tile turn
// counter (no atomics on dw), so dw is deterministic too.
#include <cuda_bf16.h>
#include <cuda_runtime.h>

#include <algorithm>

#include "mucudnn_internal.h"

namespace mucu {

namespace {

constexpr int kThreads = 256;

__device__ __forceinline__ float to_float(float v) { return v; }
__device__ __forceinline__ float to_float(__nv_bfloat16 v) { return __bfloat162float(v); }
template <class T> __device__ __forceinline__ T from_float(float v);
template <> __device__ __forceinline__ float from_float<float>(float v) { return v; }
template <> __device__ __forceinline__ __nv_bfloat16 from_float<__nv_bfloat16>(float v) { return __float2bfloat16_rn(v); }

// ------------------------------------------------------------------ views --
// Dense matrix view: A(i,kk) = p[i*si + kk*sk] (zero outside rows x kdim).
struct Dense {
    const float* p;
    int64_t rows, kdim, si, sk, batch_stride;
    // row-contiguous loads: a thread keeps one row for the whole main loop
    struct Row { const float* q; bool ok; };
    __device__ __forceinline__ Row row(int64_t i) const { return Row{p + i * si, i < rows}; }
    __device__ __forceinline__ void batch(int z) { p += z * batch_stride; }
    // k-contiguous loader contexts: a row pointer per thread row, nothing per kk
    struct KRow { const float* q; bool ok; };
    struct KCol { };
    __device__ __forceinline__ KRow krow(int64_t i) const { return KRow{p + i * si, i < rows}; }
    __device__ __forceinline__ KCol kcol(int64_t) const { return KCol{}; }
    __device__ __forceinline__ void at4c(const KRow& r, const KCol&, int64_t kk, int64_t kend, float (&o)[4]) const {
        const float* q = r.q + kk * sk;
        if (sk == 1 && r.ok && kk + 3 < kdim && kk + 3 < kend && (((uintptr_t)q) & 15) == 0) {
            const float4 v = __ldg(reinterpret_cast<const float4*>(q));
            o[0] = v.x; o[1] = v.y; o[2] = v.z; o[3] = v.w;
            return;
        }
#pragma unroll
        for (int e = 0; e < 4; ++e) o[e] = (r.ok && kk + e < kend && kk + e < kdim) ? __ldg(q + e * sk) : 0.f;
    }
    // row-contiguous loader: CNT values of the thread's row at kk0, kk0 + step, ...
    template <int CNT>
    __device__ __forceinline__ void run(const Row& r, int64_t kk0, int step, int64_t kend, float (&o)[CNT]) const {
#pragma unroll
        for (int e = 0; e < CNT; ++e) {
            const int64_t kk = kk0 + (int64_t)e * step;
            o[e] = (r.ok && kk < kend && kk < kdim) ? __ldg(r.q + kk * sk) : 0.f;
        }
    }
};

// Implicit im2col of x (NHWC) for FWD: row i = output pixel (n,p,q), kk = (r,s,c).
// Index arithmetic by multiply-high division (FastDiv): ~3 instructions per
// quotient instead of a ~20-instruction integer division per element.
struct Im2col {
    const float* x;
    int64_t rows;
    int H, W, C, P, Q, S, pad, st, RSC;
    FastDiv dPQ, dQ, dC, dS;
    __device__ __forceinline__ float at(int64_t m64, int64_t kk64) const {
        if (m64 >= rows || kk64 >= RSC) return 0.f;
        const uint32_t m = (uint32_t)m64, kk = (uint32_t)kk64;
        const uint32_t n = dPQ.div(m), rem = m - n * (uint32_t)(P * Q);
        const uint32_t p = dQ.div(rem), q = rem - p * (uint32_t)Q;
        const uint32_t rs = dC.div(kk), c = kk - rs * (uint32_t)C;
        const uint32_t r = dS.div(rs), s = rs - r * (uint32_t)S;
        const int h = (int)(p * st + r) - pad, w = (int)(q * st + s) - pad;
        if ((unsigned)h >= (unsigned)H || (unsigned)w >= (unsigned)W) return 0.f;
        return __ldg(x + (((int64_t)n * H + h) * W + w) * C + c);
    }
    __device__ __forceinline__ void batch(int) {}
    // k-contiguous loader contexts: the pixel of a thread row is decomposed once per
    // CTA, the tap (r, s, c) of the thread's kk once per K slab (shared by its rows)
    struct KRow { const float* xn; int h0, w0, m; };
    struct KCol { int r, s, c; };
    __device__ __forceinline__ KRow krow(int64_t m64) const {
        if (m64 >= rows) return KRow{x, 0, 0, -1};
        const uint32_t m = (uint32_t)m64;
        const uint32_t n = dPQ.div(m), rem = m - n * (uint32_t)(P * Q);
        const uint32_t p = dQ.div(rem), q = rem - p * (uint32_t)Q;
        return KRow{x + (int64_t)n * H * W * C, (int)(p * st) - pad, (int)(q * st) - pad, (int)m};
    }
    __device__ __forceinline__ KCol kcol(int64_t kk64) const {
        if (kk64 >= RSC) return KCol{0, 0, C};
        const uint32_t kk = (uint32_t)kk64, rs = dC.div(kk), c = kk - rs * (uint32_t)C;
        const uint32_t r = dS.div(rs), s = rs - r * (uint32_t)S;
        return KCol{(int)r, (int)s, (int)c};
    }
    __device__ __forceinline__ void at4c(const KRow& kr, const KCol& kc, int64_t kk, int64_t kend,
                                         float (&o)[4]) const {
        if (kr.m < 0) { o[0] = o[1] = o[2] = o[3] = 0.f; return; }
        if (kk + 3 < RSC && kk + 3 < kend && kc.c + 3 < C) {
            const int h = kr.h0 + kc.r, w = kr.w0 + kc.s;
            if ((unsigned)h >= (unsigned)H || (unsigned)w >= (unsigned)W) { o[0] = o[1] = o[2] = o[3] = 0.f; return; }
            const float* src = kr.xn + ((int64_t)h * W + w) * C + kc.c;
            if ((((uintptr_t)src) & 15) == 0) {
                const float4 v = __ldg(reinterpret_cast<const float4*>(src));
                o[0] = v.x; o[1] = v.y; o[2] = v.z; o[3] = v.w;
            } else {
#pragma unroll
                for (int e = 0; e < 4; ++e) o[e] = __ldg(src + e);
            }
            return;
        }
#pragma unroll
        for (int e = 0; e < 4; ++e) o[e] = kk + e < kend ? at(kr.m, kk + e) : 0.f;
    }
};
Im2col make_im2col(const float* x, int64_t rows, const Geom& g) {
    return Im2col{x, rows, g.h, g.w, g.c, g.p, g.q, g.s, g.pad, g.stride, g.r * g.s * g.c,
                  FastDiv((uint32_t)(g.p * g.q)), FastDiv((uint32_t)g.q), FastDiv((uint32_t)g.c), FastDiv((uint32_t)g.s)};
}

// Im2col transposed for WGRAD's B operand: B(j, kk) = im2col(kk = pixel, j = (r,s,c)).
struct Im2colT {
    Im2col v;
    // the (r,s,c) of a thread's row is decomposed once; each pixel then costs two divisions
    struct Row { const float* xc; int r, s; bool ok; };
    __device__ __forceinline__ Row row(int64_t j64) const {
        if (j64 >= v.RSC) return Row{v.x, 0, 0, false};
        const uint32_t j = (uint32_t)j64, rs = v.dC.div(j), c = j - rs * (uint32_t)v.C;
        const uint32_t r = v.dS.div(rs), s = rs - r * (uint32_t)v.S;
        return Row{v.x + c, (int)r - v.pad, (int)s - v.pad, true};
    }
    // CNT pixels m0, m0 + step, ...: one decomposition, then an incremental walk
    template <int CNT>
    __device__ __forceinline__ void run(const Row& rw, int64_t m0, int step, int64_t kend, float (&o)[CNT]) const {
        const int64_t lim = min(kend, v.rows);
        if (!rw.ok || m0 >= lim) {
#pragma unroll
            for (int e = 0; e < CNT; ++e) o[e] = 0.f;
            return;
        }
        const uint32_t m = (uint32_t)m0;
        uint32_t n = v.dPQ.div(m);
        const uint32_t rem = m - n * (uint32_t)(v.P * v.Q);
        uint32_t p = v.dQ.div(rem), q = rem - p * (uint32_t)v.Q;
        const float* xn = rw.xc + (int64_t)n * v.H * v.W * v.C;
        const int left = (int)(lim - m0);  // valid pixels from m0 on
#pragma unroll
        for (int e = 0; e < CNT; ++e) {
            float val = 0.f;
            const int h = (int)(p * v.st) + rw.r, w = (int)(q * v.st) + rw.s;
            if (e * step < left && (unsigned)h < (unsigned)v.H && (unsigned)w < (unsigned)v.W)
                val = __ldg(xn + (h * v.W + w) * v.C);
            o[e] = val;
            q += step;
            while (q >= (uint32_t)v.Q) {
                q -= v.Q;
                if (++p == (uint32_t)v.P) { p = 0; xn += v.H * v.W * v.C; }
            }
        }
    }
};

// DGRAD gather of dy: row i = dx pixel (n,h,w), kk = (r,s,k):
// dy[n, (h+pad-r)/st, (w+pad-s)/st, k] when st divides and in range, else 0.
struct DgradGather {
    const float* dy;
    int64_t rows;
    int H, W, K, P, Q, S, pad, st, RSK;
    FastDiv dHW, dW, dK, dS, dSt;
    __device__ __forceinline__ float at(int64_t m64, int64_t kk64) const {
        if (m64 >= rows || kk64 >= RSK) return 0.f;
        const uint32_t m = (uint32_t)m64, kk = (uint32_t)kk64;
        const uint32_t n = dHW.div(m), rem = m - n * (uint32_t)(H * W);
        const uint32_t h = dW.div(rem), w = rem - h * (uint32_t)W;
        const uint32_t rs = dK.div(kk), k = kk - rs * (uint32_t)K;
        const uint32_t r = dS.div(rs), s = rs - r * (uint32_t)S;
        const int ph = (int)(h + pad) - (int)r, pw = (int)(w + pad) - (int)s;
        if (ph < 0 || pw < 0) return 0.f;
        const uint32_t p = dSt.div((uint32_t)ph), q = dSt.div((uint32_t)pw);
        if (p * st != (uint32_t)ph || q * st != (uint32_t)pw || p >= (uint32_t)P || q >= (uint32_t)Q) return 0.f;
        return __ldg(dy + (((int64_t)n * P + p) * Q + q) * K + k);
    }
    __device__ __forceinline__ void batch(int) {}
    // k-contiguous loader contexts (see Im2col)
    struct KRow { const float* dyn; int hp, wp, m; };
    struct KCol { int r, s, k; };
    __device__ __forceinline__ KRow krow(int64_t m64) const {
        if (m64 >= rows) return KRow{dy, 0, 0, -1};
        const uint32_t m = (uint32_t)m64;
        const uint32_t n = dHW.div(m), rem = m - n * (uint32_t)(H * W);
        const uint32_t h = dW.div(rem), w = rem - h * (uint32_t)W;
        return KRow{dy + (int64_t)n * P * Q * K, (int)h + pad, (int)w + pad, (int)m};
    }
    __device__ __forceinline__ KCol kcol(int64_t kk64) const {
        if (kk64 >= RSK) return KCol{0, 0, K};
        const uint32_t kk = (uint32_t)kk64, rs = dK.div(kk), k = kk - rs * (uint32_t)K;
        const uint32_t r = dS.div(rs), s = rs - r * (uint32_t)S;
        return KCol{(int)r, (int)s, (int)k};
    }
    __device__ __forceinline__ void at4c(const KRow& kr, const KCol& kc, int64_t kk, int64_t kend,
                                         float (&o)[4]) const {
        if (kr.m < 0) { o[0] = o[1] = o[2] = o[3] = 0.f; return; }
        if (kk + 3 < RSK && kk + 3 < kend && kc.k + 3 < K) {
            o[0] = o[1] = o[2] = o[3] = 0.f;
            const int ph = kr.hp - kc.r, pw = kr.wp - kc.s;
            if (ph < 0 || pw < 0) return;
            uint32_t p = (uint32_t)ph, q = (uint32_t)pw;
            if (st != 1) {
                p = dSt.div((uint32_t)ph); q = dSt.div((uint32_t)pw);
                if (p * st != (uint32_t)ph || q * st != (uint32_t)pw) return;
            }
            if (p >= (uint32_t)P || q >= (uint32_t)Q) return;
            const float* src = kr.dyn + ((int64_t)p * Q + q) * K + kc.k;
            if ((((uintptr_t)src) & 15) == 0) {
                const float4 v = __ldg(reinterpret_cast<const float4*>(src));
                o[0] = v.x; o[1] = v.y; o[2] = v.z; o[3] = v.w;
            } else {
#pragma unroll
                for (int e = 0; e < 4; ++e) o[e] = __ldg(src + e);
            }
            return;
        }
#pragma unroll
        for (int e = 0; e < 4; ++e) o[e] = kk + e < kend ? at(kr.m, kk + e) : 0.f;
    }
};

// DGRAD filter view: B(j = c, kk = (r,s,k)) = w[k][r][s][c].
struct DgradFilter {
    const float* w;
    int C, K, RS;
    FastDiv dK;
    struct Row { const float* q; bool ok; };
    __device__ __forceinline__ Row row(int64_t j) const { return Row{w + j, j < C}; }
    // CNT taps kk0, kk0 + step, ...: one decomposition, then an incremental walk
    template <int CNT>
    __device__ __forceinline__ void run(const Row& r, int64_t kk0, int step, int64_t kend, float (&o)[CNT]) const {
        const int64_t lim = min(kend, (int64_t)RS * K);
        uint32_t rs = 0, k = 0;
        if (kk0 < lim) { rs = dK.div((uint32_t)kk0); k = (uint32_t)kk0 - rs * (uint32_t)K; }
#pragma unroll
        for (int e = 0; e < CNT; ++e) {
            o[e] = (r.ok && kk0 + (int64_t)e * step < lim) ? __ldg(r.q + ((int64_t)k * RS + rs) * C) : 0.f;
            k += step;
            while (k >= (uint32_t)K) { k -= K; ++rs; }
        }
    }
    __device__ __forceinline__ void batch(int) {}
};

// -------------------------------------------------------------- epilogues --
struct StoreDense {
    float* c;
    int64_t rows, cols, ldc, batch_stride;
    float alpha, beta;
    __device__ __forceinline__ void batch(int z) { c += z * batch_stride; }
    template <int TN>
    __device__ __forceinline__ void row(int64_t i, int64_t j0, const float (&v)[TN]) const {
        if (i >= rows) return;
        float* dst = c + i * ldc;
#pragma unroll
        for (int j = 0; j < TN; ++j) {
            int64_t jj = j0 + j;
            if (jj < cols) {
                float o = alpha * v[j];
                if (beta != 0.f) o += beta * dst[jj];
                dst[jj] = o;
            }
        }
    }
};

// ------------------------------------------------------------ the kernel --
// CONTIG_A / CONTIG_B: true when consecutive kk are contiguous in memory
// (threads of a warp then spread along kk), false when consecutive rows are.
// K slab per pipeline step: 16 (two FFMA blocks of 8 between barriers).
constexpr int kBK = 16;

// row context of a row-contiguous operand (views without one are only loaded k-contiguous)
template <class V, bool CONTIG> struct RowOf { using type = typename V::Row; };
template <class V> struct RowOf<V, true> { using type = int; };
template <class V, bool CONTIG> struct KRowOf { using type = int; };
template <class V> struct KRowOf<V, true> { using type = typename V::KRow; };

template <int BM, int BN, bool CONTIG_KA, bool CONTIG_KB, class AV, class BV>
struct TileLoader {
    static constexpr int BK = kBK;
    static constexpr int NA = BM * BK / kThreads;
    static constexpr int NB = BN * BK / kThreads;
    float ra[NA], rb[NB];
    typename RowOf<AV, CONTIG_KA>::type arow;  // row-contiguous: the thread's row is fixed (t % BM)
    typename RowOf<BV, CONTIG_KB>::type brow;
    // k-contiguous: the thread's NA / 4 (NB / 4) rows are fixed too -- their contexts
    // (pixel decompositions) are computed once per CTA
    typename KRowOf<AV, CONTIG_KA>::type akr[CONTIG_KA ? NA / 4 : 1];
    typename KRowOf<BV, CONTIG_KB>::type bkr[CONTIG_KB ? NB / 4 : 1];

    __device__ __forceinline__ void init(const AV& a, const BV& b, int64_t m0, int64_t n0) {
        if constexpr (!CONTIG_KA) arow = a.row(m0 + threadIdx.x % BM);
        if constexpr (!CONTIG_KB) brow = b.row(n0 + threadIdx.x % BN);
        if constexpr (CONTIG_KA) {
#pragma unroll
            for (int g = 0; g < NA / 4; ++g) { int il, kl; a_coord(4 * g, il, kl); akr[g] = a.krow(m0 + il); }
        }
        if constexpr (CONTIG_KB) {
#pragma unroll
            for (int g = 0; g < NB / 4; ++g) { int jl, kl; b_coord(4 * g, jl, kl); bkr[g] = b.krow(n0 + jl); }
        }
    }

    // k-contiguous operands: a thread loads 4 consecutive k of a row (element e = 4g + u:
    // group g of rows, k offset 4*(t % (BK/4)) + u); row-contiguous: one k per element.
    __device__ __forceinline__ static void a_coord(int e, int& il, int& kl) {
        const int t = threadIdx.x;
        if (CONTIG_KA) { kl = 4 * (t % (BK / 4)) + (e & 3); il = t / (BK / 4) + (e >> 2) * (kThreads * 4 / BK); }
        else           { il = t % BM; kl = t / BM + e * (kThreads / BM); }
    }
    __device__ __forceinline__ static void b_coord(int e, int& jl, int& kl) {
        const int t = threadIdx.x;
        if (CONTIG_KB) { kl = 4 * (t % (BK / 4)) + (e & 3); jl = t / (BK / 4) + (e >> 2) * (kThreads * 4 / BK); }
        else           { jl = t % BN; kl = t / BN + e * (kThreads / BN); }
    }
    __device__ __forceinline__ void load(const AV& a, const BV& b, int64_t, int64_t, int64_t k0, int64_t kend) {
        if constexpr (CONTIG_KA) {
            // every group of the thread reads the same 4 kk: one tap decomposition
            const int64_t kk = k0 + 4 * (threadIdx.x % (BK / 4));
            const typename AV::KCol kc = a.kcol(kk);
#pragma unroll
            for (int g = 0; g < NA / 4; ++g) {
                float o[4];
                a.at4c(akr[g], kc, kk, kend, o);
#pragma unroll
                for (int u = 0; u < 4; ++u) ra[4 * g + u] = o[u];
            }
        } else {
            a.template run<NA>(arow, k0 + threadIdx.x / BM, kThreads / BM, kend, ra);
        }
        if constexpr (CONTIG_KB) {
            const int64_t kk = k0 + 4 * (threadIdx.x % (BK / 4));
            const typename BV::KCol kc = b.kcol(kk);
#pragma unroll
            for (int g = 0; g < NB / 4; ++g) {
                float o[4];
                b.at4c(bkr[g], kc, kk, kend, o);
#pragma unroll
                for (int u = 0; u < 4; ++u) rb[4 * g + u] = o[u];
            }
        } else {
            b.template run<NB>(brow, k0 + threadIdx.x / BN, kThreads / BN, kend, rb);
        }
    }
    __device__ __forceinline__ void store(float (*As)[BM + 4], float (*Bs)[BN + 4]) const {
#pragma unroll
        for (int e = 0; e < NA; ++e) { int il, kl; a_coord(e, il, kl); As[kl][il] = ra[e]; }
#pragma unroll
        for (int e = 0; e < NB; ++e) { int jl, kl; b_coord(e, jl, kl); Bs[kl][jl] = rb[e]; }
    }
};

// Resident CTAs per SM the register budget is pinned to (64 x 64: 4 x 256 threads x
// 64 registers; larger tiles: 2 x 256 x 128).
constexpr int ctas_per_sm(int bm, int bn) { return bm * bn <= 64 * 64 ? 4 : 2; }

// Thread tile: TM x TN outputs; with 8 they are two 4-wide blocks half a tile apart
// (rows ty*4 + i and BM/2 + ty*4 + i), so a warp's 16 tx read 16 consecutive float4
// of a shared-memory row (2 wavefronts, no bank conflicts) instead of 16 float4 at a
// 32-byte stride (4-way conflicts).
template <int T, int B>
__device__ __forceinline__ int frag_off(int t, int i) {
    if constexpr (T == 8) return t * 4 + (i & 3) + (i >> 2) * (B / 2);
    else return t * T + i;
}

// Main loop shared by all SIMT contractions: accumulates the BM x BN tile at
// (m0, n0) over kk in [kbeg, kend).  acc[i][j] belongs to row frag_off<TM,BM>(ty, i),
// column frag_off<TN,BN>(tx, j) of the tile.
template <int BM, int BN, bool CKA, bool CKB, class AV, class BV>
__device__ __forceinline__ void simt_mainloop(const AV& a, const BV& b, int64_t m0, int64_t n0, int64_t kbeg,
                                              int64_t kend, float (&acc)[BM / 16][BN / 16]) {
    constexpr int BK = kBK, TM = BM / 16, TN = BN / 16;
    __shared__ __align__(16) float As[2][BK][BM + 4];
    __shared__ __align__(16) float Bs[2][BK][BN + 4];
    const int tx = threadIdx.x % 16, ty = threadIdx.x / 16;
#pragma unroll
    for (int i = 0; i < TM; ++i)
#pragma unroll
        for (int j = 0; j < TN; ++j) acc[i][j] = 0.f;
    if (kbeg >= kend) return;
    TileLoader<BM, BN, CKA, CKB, AV, BV> ld;
    ld.init(a, b, m0, n0);
    ld.load(a, b, m0, n0, kbeg, kend);
    ld.store(As[0], Bs[0]);
    __syncthreads();
    int buf = 0;
    for (int64_t k0 = kbeg; k0 < kend; k0 += BK) {
        const bool more = k0 + BK < kend;
        if (more) ld.load(a, b, m0, n0, k0 + BK, kend);
#pragma unroll
        for (int k = 0; k < BK; ++k) {
            float af[TM], bf[TN];
#pragma unroll
            for (int i = 0; i < TM; i += 4) {
                float4 v = *reinterpret_cast<const float4*>(&As[buf][k][frag_off<TM, BM>(ty, i)]);
                af[i] = v.x; af[i + 1] = v.y; af[i + 2] = v.z; af[i + 3] = v.w;
            }
#pragma unroll
            for (int j = 0; j < TN; j += 4) {
                float4 v = *reinterpret_cast<const float4*>(&Bs[buf][k][frag_off<TN, BN>(tx, j)]);
                bf[j] = v.x; bf[j + 1] = v.y; bf[j + 2] = v.z; bf[j + 3] = v.w;
            }
#pragma unroll
            for (int i = 0; i < TM; ++i)
#pragma unroll
                for (int j = 0; j < TN; ++j) acc[i][j] = fmaf(af[i], bf[j], acc[i][j]);
        }
        if (more) ld.store(As[buf ^ 1], Bs[buf ^ 1]);
        __syncthreads();
        buf ^= 1;
    }
}

template <int BM, int BN, bool CKA, bool CKB, class AV, class BV, class EPI>
__global__ void __launch_bounds__(kThreads, ctas_per_sm(BM, BN)) simt_gemm_kernel(AV a, BV b, EPI epi, int64_t Kd) {
    constexpr int TM = BM / 16, TN = BN / 16;
    a.batch(blockIdx.z); b.batch(blockIdx.z); epi.batch(blockIdx.z);
    const int64_t m0 = (int64_t)blockIdx.x * BM, n0 = (int64_t)blockIdx.y * BN;  // M on grid.x (no 65535 cap)
    float acc[TM][TN];
    simt_mainloop<BM, BN, CKA, CKB>(a, b, m0, n0, 0, Kd, acc);
    const int tx = threadIdx.x % 16, ty = threadIdx.x / 16;
#pragma unroll
    for (int i = 0; i < TM; ++i)
#pragma unroll
        for (int j = 0; j < TN; j += 4)
            epi.template row<4>(m0 + frag_off<TM, BM>(ty, i), n0 + frag_off<TN, BN>(tx, j),
                                *reinterpret_cast<const float(*)[4]>(&acc[i][j]));
}

// WGRAD: dw[K][RSC] (+)= alpha * sum over the split's pixel range.  Splits of
// one tile are combined in split order (turns.cu): split s waits until the
// tile's counter holds tag(epoch, s-1), adds its partial (split 0 applies
// beta) and publishes tag(epoch, s).  blockIdx.z = split, so all CTAs of split
// s are dispatched before any of split s + 1 (no deadlock).
template <int BM, int BN, class AV, class BV>
__global__ void __launch_bounds__(kThreads, ctas_per_sm(BM, BN)) simt_wgrad_kernel(AV a, BV b, float* dw, int64_t rows, int64_t cols,
                                                              int64_t Kd, int64_t k_per_split, float alpha,
                                                              float beta, unsigned long long* turns,
                                                              unsigned long long epoch) {
    constexpr int TM = BM / 16, TN = BN / 16;
    const int64_t m0 = (int64_t)blockIdx.x * BM, n0 = (int64_t)blockIdx.y * BN;
    const int split = blockIdx.z, nsplit = gridDim.z;
    const int64_t kb = (int64_t)split * k_per_split;
    const int64_t ke = min(Kd, kb + k_per_split);
    float acc[TM][TN];
    simt_mainloop<BM, BN, false, false>(a, b, m0, n0, kb, ke, acc);
    const int tile = blockIdx.y * gridDim.x + blockIdx.x;
    if (threadIdx.x == 0 && split > 0) turn_wait(turns + tile, turn_tag(epoch, split - 1));
    __syncthreads();
    const int tx = threadIdx.x % 16, ty = threadIdx.x / 16;
    // the hand-off is on the ordered chain's critical path: every load of the thread's
    // TM x TN elements is issued before the first store (one L2 round trip, not TM x TN)
    const float bs = split > 0 ? 1.f : beta;
    if (bs != 0.f) {
#pragma unroll
        for (int i = 0; i < TM; ++i) {
            const int64_t r = m0 + frag_off<TM, BM>(ty, i);
#pragma unroll
            for (int j = 0; j < TN; ++j) {
                const int64_t cidx = n0 + frag_off<TN, BN>(tx, j);
                acc[i][j] = alpha * acc[i][j];
                if (r < rows && cidx < cols) acc[i][j] += bs * __ldcg(dw + r * cols + cidx);
            }
        }
    } else {
#pragma unroll
        for (int i = 0; i < TM; ++i)
#pragma unroll
            for (int j = 0; j < TN; ++j) acc[i][j] = alpha * acc[i][j];
    }
#pragma unroll
    for (int i = 0; i < TM; ++i) {
        const int64_t r = m0 + frag_off<TM, BM>(ty, i);
        if (r >= rows) continue;
#pragma unroll
        for (int j = 0; j < TN; ++j) {
            const int64_t cidx = n0 + frag_off<TN, BN>(tx, j);
            if (cidx < cols) dw[r * cols + cidx] = acc[i][j];
        }
    }
    __syncthreads();
    if (threadIdx.x == 0 && split + 1 < nsplit) turn_post(turns + tile, turn_tag(epoch, split));
}

template <int BM, int BN, bool CKA, bool CKB, class AV, class BV, class EPI>
int launch_gemm(const AV& a, const BV& b, const EPI& e, int64_t M, int64_t N, int64_t Kd, int batch,
                cudaStream_t st) {
    dim3 grid((unsigned)ceil_div(M, BM), (unsigned)ceil_div(N, BN), (unsigned)batch);
    simt_gemm_kernel<BM, BN, CKA, CKB><<<grid, kThreads, 0, st>>>(a, b, e, Kd);
    count_launch();
    return (int)cudaGetLastError();
}

// Tile shape: whole waves of CTAs over the SMs (ctas_per_sm resident CTAs) weighted by the FFMA efficiency of the thread tile
// (8 x 8 > 8 x 4 > 4 x 4 outputs per thread per shared-memory load); small GEMMs
// (cfg1: AlexNet conv2 at N = 8, 5832 x 192) take the smaller tiles.
template <bool CKA, bool CKB, class AV, class BV, class EPI>
int dispatch_gemm(const AV& a, const BV& b, const EPI& e, int64_t M, int64_t N, int64_t Kd, int batch,
                  cudaStream_t st) {
    static int sms = 0;
    if (!sms) {
        int dev = 0;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
        if (sms <= 0) sms = 148;
    }
    struct Cand { int bm, bn, per_sm; double eff; };
    const Cand cands[3] = {{128, 128, ctas_per_sm(128, 128), 1.0}, {128, 64, ctas_per_sm(128, 64), 0.9},
                           {64, 64, ctas_per_sm(64, 64), 0.75}};
    int best = 0;
    double best_cost = 1e300;
    for (int i = 0; i < 3; ++i) {
        const Cand& c = cands[i];
        if (N <= 64 && c.bn == 128) continue;
        const int64_t tiles = ceil_div(M, c.bm) * ceil_div(N, c.bn) * batch;
        const double cost = (double)ceil_div(tiles, (int64_t)sms * c.per_sm) * c.per_sm * c.bm * c.bn / c.eff;
        if (cost < best_cost - 1e-9) { best_cost = cost; best = i; }
    }
    if (best == 0) return launch_gemm<128, 128, CKA, CKB>(a, b, e, M, N, Kd, batch, st);
    if (best == 1) return launch_gemm<128, 64, CKA, CKB>(a, b, e, M, N, Kd, batch, st);
    return launch_gemm<64, 64, CKA, CKB>(a, b, e, M, N, Kd, batch, st);
}

// ------------------------------------------- small-C BackwardData (FFMA) --
// dx of a layer with C <= 4 input channels (the RGB layer) is a contraction with
// N = C output columns: no tensor-core tile fits it.  Phase decomposition
// (P:L56 BackwardData = transposed convolution): dx pixels with
// (h + pad) % st == a and (w + pad) % st == b0 receive only the taps
// r = a + st*i, s = b0 + st*j, from dy pixel (hh - i, ww - j) of the phase
// sub-grid (h = a - pad + st*hh).  One CTA = a 16 x 16 block of one phase
// sub-grid of one image: the dy block it reads ((16+nr-1) x (16+ns-1) pixels x K,
// fp32, row pitch K+4) and the phase's sub-filter [i][j][k][4] are staged in
// shared memory (each dy element is reused by up to nr*ns pixels); one thread =
// one dx pixel, all C channels, fp32 FFMA over (i, j, k) with 16-byte shared
// loads.  The sum order over (i, j, k) is fixed: independent of the micro-batch
// size (I1).
template <class T>
__global__ void __launch_bounds__(256) small_c_dgrad_kernel(const T* __restrict__ dy, const T* __restrict__ w, T* dx,
                                                            int H, int W, int C, int K, int P, int Q, int R, int S,
                                                            int pad, int st, float alpha, float beta) {
    extern __shared__ __align__(16) float sm[];
    const int a = blockIdx.y / st, b0 = blockIdx.y - (blockIdx.y / st) * st;
    const int n = blockIdx.z;
    const int nr = a < R ? (R - a + st - 1) / st : 0, ns = b0 < S ? (S - b0 + st - 1) / st : 0;
    const int KP = K + 4, BR = 16 + nr - 1, BC = 16 + ns - 1;
    float* dys = sm;                               // [BR][BC][KP]
    float* wsm = sm + (size_t)BR * BC * KP;        // [nr][ns][K][4]
    const int hh0 = (pad - a + st - 1) / st > 0 ? (pad - a + st - 1) / st : 0;  // first h >= 0
    const int ww0 = (pad - b0 + st - 1) / st > 0 ? (pad - b0 + st - 1) / st : 0;
    const int tiles_w = (W + st - 1) / st / 16 + 1;
    const int hb = hh0 + (blockIdx.x / tiles_w) * 16, wb = ww0 + (blockIdx.x % tiles_w) * 16;
    // the phase's sub-filter, channels padded to 4
    for (int idx = threadIdx.x; idx < nr * ns * K * 4; idx += 256) {
        const int c = idx & 3, t = idx >> 2, k = t % K, t2 = t / K, jj = t2 % ns, ii = t2 / ns;
        wsm[idx] = c < C ? to_float(w[(((size_t)k * R + a + st * ii) * S + b0 + st * jj) * C + c]) : 0.f;
    }
    // dy block: pixel (pp, qq) = (hb - (nr-1) + row, wb - (ns-1) + col), zero outside dy
    for (int idx = threadIdx.x; idx < BR * BC * (K / 4); idx += 256) {
        const int k4 = idx % (K / 4), t = idx / (K / 4), col = t % BC, row = t / BC;
        const int pp = hb - (nr - 1) + row, qq = wb - (ns - 1) + col;
        float4 v = make_float4(0.f, 0.f, 0.f, 0.f);
        if (pp >= 0 && pp < P && qq >= 0 && qq < Q) {
            const T* d = dy + (((size_t)n * P + pp) * Q + qq) * K + 4 * k4;
            v = make_float4(to_float(d[0]), to_float(d[1]), to_float(d[2]), to_float(d[3]));
        }
        *reinterpret_cast<float4*>(dys + ((size_t)row * BC + col) * KP + 4 * k4) = v;
    }
    __syncthreads();
    const int ty = threadIdx.x / 16, tx = threadIdx.x % 16;
    const int hh = hb + ty, ww = wb + tx;
    const int h = a - pad + st * hh, x = b0 - pad + st * ww;
    if (h >= H || x >= W) return;
    float acc[4] = {0.f, 0.f, 0.f, 0.f};
    for (int i = 0; i < nr; ++i) {
        for (int j = 0; j < ns; ++j) {
            const float* d = dys + ((size_t)(ty + nr - 1 - i) * BC + (tx + ns - 1 - j)) * KP;
            const float* wf = wsm + (size_t)(i * ns + j) * K * 4;
            for (int k = 0; k < K; k += 4) {
                const float4 v = *reinterpret_cast<const float4*>(d + k);
                const float vv[4] = {v.x, v.y, v.z, v.w};
#pragma unroll
                for (int u = 0; u < 4; ++u) {
                    const float4 f = *reinterpret_cast<const float4*>(wf + (k + u) * 4);
                    acc[0] = fmaf(vv[u], f.x, acc[0]);
                    acc[1] = fmaf(vv[u], f.y, acc[1]);
                    acc[2] = fmaf(vv[u], f.z, acc[2]);
                    acc[3] = fmaf(vv[u], f.w, acc[3]);
                }
            }
        }
    }
    T* o = dx + (((size_t)n * H + h) * W + x) * C;
#pragma unroll
    for (int c = 0; c < 4; ++c) {
        if (c >= C) break;
        float r = alpha * acc[c];
        if (beta != 0.f) r += beta * to_float(o[c]);
        o[c] = from_float<T>(r);
    }
}

}  // namespace

int small_c_dgrad(const Geom& g, int32_t b, float alpha, const void* dy, const void* w, float beta, void* dx,
                  cudaStream_t st) {
    if (g.c > 4 || g.k % 4) return -1;
    const int nr = (g.r + g.stride - 1) / g.stride, ns = (g.s + g.stride - 1) / g.stride;
    const size_t smem = ((size_t)(16 + nr - 1) * (16 + ns - 1) * (g.k + 4) + (size_t)nr * ns * g.k * 4) * sizeof(float);
    if (smem > 220 * 1024) return -1;
    const int tiles_h = (g.h + g.stride - 1) / g.stride / 16 + 1, tiles_w = (g.w + g.stride - 1) / g.stride / 16 + 1;
    dim3 grid((unsigned)(tiles_h * tiles_w), (unsigned)(g.stride * g.stride), (unsigned)b);
    if (g.math == MUCU_MATH_BF16) {
        auto k = small_c_dgrad_kernel<__nv_bfloat16>;
        cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        k<<<grid, 256, smem, st>>>((const __nv_bfloat16*)dy, (const __nv_bfloat16*)w, (__nv_bfloat16*)dx, g.h, g.w,
                                   g.c, g.k, g.p, g.q, g.r, g.s, g.pad, g.stride, alpha, beta);
    } else {
        auto k = small_c_dgrad_kernel<float>;
        cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        k<<<grid, 256, smem, st>>>((const float*)dy, (const float*)w, (float*)dx, g.h, g.w, g.c, g.k, g.p, g.q,
                                   g.r, g.s, g.pad, g.stride, alpha, beta);
    }
    count_launch();
    return (int)cudaGetLastError();
}

// FWD implicit GEMM (algorithm (a)): y[m][k] = sum_{(r,s,c)} im2col(x)[m][(r,s,c)] * w[k][(r,s,c)].
int simt_fwd_ig(const Geom& g, int32_t b, float alpha, const float* x, const float* w, float beta, float* y,
                cudaStream_t st) {
    const int64_t M = (int64_t)b * g.p * g.q, N = g.k, Kd = (int64_t)g.r * g.s * g.c;
    Im2col a = make_im2col(x, M, g);
    Dense bw{w, N, Kd, Kd, 1, 0};
    StoreDense e{y, M, N, N, 0, alpha, beta};
    return dispatch_gemm<true, true>(a, bw, e, M, N, Kd, 1, st);
}

// C[M,N] = alpha * A[M,K] * B[N,K]^T + beta * C, optional batch (strides in elements).
int simt_gemm_nt(int64_t M, int64_t N, int64_t K, float alpha, const float* A, int64_t lda, const float* B,
                 int64_t ldb, float beta, float* C, int64_t ldc, int batch, int64_t sA, int64_t sB, int64_t sC,
                 cudaStream_t st) {
    Dense a{A, M, K, lda, 1, sA};
    Dense bb{B, N, K, ldb, 1, sB};
    StoreDense e{C, M, N, ldc, sC, alpha, beta};
    return dispatch_gemm<true, true>(a, bb, e, M, N, K, batch, st);
}

// C[M,N] = alpha * A[M,K] * B[K,N] + beta * C (B row-major, N contiguous).
int simt_gemm_nn(int64_t M, int64_t N, int64_t K, float alpha, const float* A, int64_t lda, const float* B,
                 int64_t ldb, float beta, float* C, int64_t ldc, cudaStream_t st) {
    Dense a{A, M, K, lda, 1, 0};
    Dense bb{B, N, K, 1, ldb, 0};
    StoreDense e{C, M, N, ldc, 0, alpha, beta};
    return dispatch_gemm<true, false>(a, bb, e, M, N, K, 1, st);
}

// DGRAD implicit GEMM: dx[m][c] = sum_{(r,s,k)} gather(dy)[m][(r,s,k)] * w[k][r][s][c].
int simt_dgrad_ig(const Geom& g, int32_t b, float alpha, const float* dy, const float* w, float beta, float* dx,
                  cudaStream_t st) {
    const int64_t M = (int64_t)b * g.h * g.w, N = g.c, Kd = (int64_t)g.r * g.s * g.k;
    DgradGather a{dy, M, g.h, g.w, g.k, g.p, g.q, g.s, g.pad, g.stride, (int)Kd, FastDiv((uint32_t)(g.h * g.w)),
                  FastDiv((uint32_t)g.w), FastDiv((uint32_t)g.k), FastDiv((uint32_t)g.s), FastDiv((uint32_t)g.stride)};
    DgradFilter bw{w, g.c, g.k, g.r * g.s, FastDiv((uint32_t)g.k)};
    StoreDense e{dx, M, N, N, 0, alpha, beta};
    return dispatch_gemm<true, false>(a, bw, e, M, N, Kd, 1, st);
}

// WGRAD: dw[k][(r,s,c)] = sum_m dy[m][k] * B(m, (r,s,c)), B = implicit im2col
// of x (IG) or the explicit col matrix (I2C, row pitch kpitch).
template <int BM, int BN>
int simt_wgrad_t(const Geom& g, int32_t b, float alpha, const float* dy, const float* xin, bool col_input,
                 int32_t kpitch, float beta, float* dw, int num_sms, cudaStream_t st) {
    constexpr int BK = kBK;
    const int64_t rows = g.k, cols = (int64_t)g.r * g.s * g.c, Kd = (int64_t)b * g.p * g.q;
    const int64_t tiles = ceil_div(cols, BN) * ceil_div(rows, BM);
    // Split count: waves of 2 CTAs per SM x pixels per split (a pixel of a BM x BN
    // tile ~ BM*BN/64 cycles at half an SM's FFMA rate) + the ordered hand-over of
    // the partial tiles (~4000 cycles per split, the deterministic chain).
    int64_t nsplit = 1;
    double best = 1e300;
    const int64_t smax = std::min<int64_t>(std::max<int64_t>(1, Kd / 64), 1024);
    for (int64_t sp = 1; sp <= smax; ++sp) {
        const double cost = (double)ceil_div(tiles * sp, 2LL * num_sms) * (double)ceil_div(Kd, sp) * (BM * BN / 64.0) +
                            (double)sp * 4000.0;
        if (cost < best) { best = cost; nsplit = sp; }
    }
    int64_t kps = ceil_div(ceil_div(Kd, nsplit), BK) * BK;
    nsplit = ceil_div(Kd, kps);
    dim3 grid((unsigned)ceil_div(rows, BM), (unsigned)ceil_div(cols, BN), (unsigned)nsplit);
    TurnRange tr{nullptr, 0};
    if (nsplit > 1) {
        const int e = alloc_turns(tiles, &tr);
        if (e) return e;
    }
    Dense a{dy, rows, Kd, 1, g.k, 0};  // A(k, m) = dy[m][k]
    if (col_input) {
        Dense bb{xin, cols, Kd, 1, kpitch, 0};  // B(j, m) = col[m][j]
        simt_wgrad_kernel<BM, BN><<<grid, kThreads, 0, st>>>(a, bb, dw, rows, cols, Kd, kps, alpha, beta, tr.ctr, tr.epoch);
    } else {
        Im2colT bb{make_im2col(xin, Kd, g)};
        simt_wgrad_kernel<BM, BN><<<grid, kThreads, 0, st>>>(a, bb, dw, rows, cols, Kd, kps, alpha, beta, tr.ctr, tr.epoch);
    }
    count_launch();
    return (int)cudaGetLastError();
}

int simt_wgrad(const Geom& g, int32_t b, float alpha, const float* dy, const float* xin, bool col_input,
               int32_t kpitch, float beta, float* dw, int num_sms, cudaStream_t st) {
    // rows = K filters: half-empty 128-row tiles for K <= 64 (AlexNet / ResNet conv1)
    if (g.k <= 64) return simt_wgrad_t<64, 128>(g, b, alpha, dy, xin, col_input, kpitch, beta, dw, num_sms, st);
    return simt_wgrad_t<128, 128>(g, b, alpha, dy, xin, col_input, kpitch, beta, dw, num_sms, st);
}

// Winograd BackwardFilter GEMMs: M[z][k][c] = sum_t D[z][t][k] * V[z][t][c], z < 16.
int simt_gemm_tt(int64_t K, int64_t C, int64_t Tp, const float* V, const float* D, float* M, int64_t ldt,
                 cudaStream_t st) {
    const int64_t Kp = (K + 31) / 32 * 32, Cp = (C + 31) / 32 * 32;  // channel pitches (128 B of fp32)
    Dense a{D, K, Tp, 1, Kp, ldt * Kp};   // A(k, t) = D[z][t][k]
    Dense bb{V, C, Tp, 1, Cp, ldt * Cp};  // B(c, t) = V[z][t][c]
    StoreDense e{M, K, C, Cp, Kp * Cp, 1.f, 0.f};
    return dispatch_gemm<false, false>(a, bb, e, K, C, Tp, 16, st);
}

}  // namespace mucu
