// kernels_fft.cu -- FFT and FFT_TILING convolution algorithms (MUCU_MATH_F32).
//
// The two workspace-hungry algorithms behind the paper's largest micro-batching
// gains: cuDNN's FFT (conv2 FWD needs 213 MiB at N = 256, 48.9 MiB at b = 32,
// P:L212 Sec. IV-A) and FFT_TILING (the top-left Pareto point of conv2 FWD,
// P:L127 Fig. 8; fastest conv5 FWD, Sec. IV-D).  Same convolution as the
// other algorithms, computed in the frequency domain; DESIGN.md 6.11.
//
// A "plane" is one F x F tile of one image: FFT uses a single tile per image
// (F = the smallest power of two >= the tile's input extent, F <= 32),
// FFT_TILING covers the output with tiles of Th x Tw = (33 - R) x (33 - S)
// outputs on a fixed F = 32 grid.  Per micro-batch:
//   1. forward real 2-D DFT of every (plane, channel) tile of the input operand
//      (zero outside the tensor) -> spectrum [bin][plane][channel], complex;
//      the filter spectrum [bin][k][c] (b-independent, once per call);
//   2. per frequency bin a complex GEMM over channels (or over planes for
//      BackwardFilter), on the CUDA cores in fp32;
//   3. inverse 2-D DFT of every (plane, channel) result tile, crop, alpha/beta.
// Circular correlation of size F equals the linear one on the cropped window
// because every tile keeps Th + R - 1 <= F (no wrap-around):
//   FWD    y  = IDFT( X . conj(W) )            window [0, Th) x [0, Tw)
//   DGRAD  dx = IDFT( DY . W ), dy tile from h0 + pad - (R-1), window from (R-1, S-1)
//   WGRAD  dw = IDFT( sum_planes X . conj(DY) ), dy zero outside its tile, window R x S
// DFTs: radix-2 decimation in time on F complex values held in registers by one
// thread (rows first, then the F/2 + 1 Hermitian-half columns), tiles staged in
// shared memory.

#include <cuda_runtime.h>

#include <algorithm>

#include "mucudnn_internal.h"

namespace mucu {

namespace {

// exp(-2 pi i k / 64), k < 32: twiddles of every power-of-two length <= 64
__constant__ float2 c_tw[32] = {
    {1.000000000f, -0.000000000f},  {0.995184727f, -0.098017140f},  {0.980785280f, -0.195090322f},
    {0.956940336f, -0.290284677f},  {0.923879533f, -0.382683432f},  {0.881921264f, -0.471396737f},
    {0.831469612f, -0.555570233f},  {0.773010453f, -0.634393284f},  {0.707106781f, -0.707106781f},
    {0.634393284f, -0.773010453f},  {0.555570233f, -0.831469612f},  {0.471396737f, -0.881921264f},
    {0.382683432f, -0.923879533f},  {0.290284677f, -0.956940336f},  {0.195090322f, -0.980785280f},
    {0.098017140f, -0.995184727f},  {0.000000000f, -1.000000000f},  {-0.098017140f, -0.995184727f},
    {-0.195090322f, -0.980785280f}, {-0.290284677f, -0.956940336f}, {-0.382683432f, -0.923879533f},
    {-0.471396737f, -0.881921264f}, {-0.555570233f, -0.831469612f}, {-0.634393284f, -0.773010453f},
    {-0.707106781f, -0.707106781f}, {-0.773010453f, -0.634393284f}, {-0.831469612f, -0.555570233f},
    {-0.881921264f, -0.471396737f}, {-0.923879533f, -0.382683432f}, {-0.956940336f, -0.290284677f},
    {-0.980785280f, -0.195090322f}, {-0.995184727f, -0.098017140f}};

template <int F> struct Log2 { static constexpr int v = 1 + Log2<F / 2>::v; };
template <> struct Log2<1> { static constexpr int v = 0; };
template <int I, int L> struct BitRev { static constexpr int v = ((I & 1) << (L - 1)) | BitRev<(I >> 1), L - 1>::v; };
template <int I> struct BitRev<I, 0> { static constexpr int v = 0; };
// bit-reversal permutation with compile-time register indices
template <int F, int I = 0>
__device__ __forceinline__ void bit_reverse_permute(float2 (&z)[F]) {
    if constexpr (I < F) {
        constexpr int J = BitRev<I, Log2<F>::v>::v;
        if constexpr (I < J) { const float2 t = z[I]; z[I] = z[J]; z[J] = t; }
        bit_reverse_permute<F, I + 1>(z);
    }
}

// One radix-2 stage (butterfly span LEN / 2) and the following ones, unrolled at
// compile time (register indices must be constants).
template <int F, bool INV, int LEN>
__device__ __forceinline__ void dft_stages(float2 (&z)[F]) {
    if constexpr (LEN <= F) {
        constexpr int half = LEN / 2, step = 64 / LEN;
#pragma unroll
        for (int i = 0; i < F; i += LEN) {
#pragma unroll
            for (int k = 0; k < half; ++k) {
                float2 w = c_tw[k * step];
                if (INV) w.y = -w.y;
                const float2 a = z[i + k], b = z[i + k + half];
                const float2 t = make_float2(b.x * w.x - b.y * w.y, b.x * w.y + b.y * w.x);
                z[i + k] = make_float2(a.x + t.x, a.y + t.y);
                z[i + k + half] = make_float2(a.x - t.x, a.y - t.y);
            }
        }
        dft_stages<F, INV, LEN * 2>(z);
    }
}

// In-register DFT of length F (unnormalised): Z[u] = sum_j z[j] exp(-+2 pi i u j / F),
// radix-2 decimation in time.
template <int F, bool INV>
__device__ __forceinline__ void dft(float2 (&z)[F]) {
    bit_reverse_permute<F>(z);
    dft_stages<F, INV, 2>(z);
}

// Source / destination of a tile transform: an NHWC tensor (filters: [K][R][S][C]
// read as N = K images of R x S pixels).  Plane p = (image n, tile ty, tx); its
// tile covers rows ty*Th + oh + [0, F) (forward: loaded where inside the tensor
// and inside the region rh x rw of the tile, else 0) or writes rows ty*Th + [0, Th)
// from the DFT window starting at (oh, ow) (inverse).
struct TileMap {
    int H, W, C;          // tensor extent (channels = the transform's channel axis)
    int tiles_x, tiles;   // tiles per image row / per image
    int Th, Tw;           // tile step (output pixels per tile)
    int oh, ow;           // forward: input origin offset; inverse: crop offset in the DFT
    int rh, rw;           // forward: load region of the tile
    int64_t planes;       // planes of the spectrum (its [bin][plane][C] pitch)
};

template <int F> struct FftCfg {
    static constexpr int CB = 256 / F;        // channels per CTA (one row DFT per thread)
    static constexpr int V = F / 2 + 1;       // Hermitian half
    static constexpr int RP = F + 1;          // real row pitch (floats)
    static constexpr int PP = F * RP + 1;     // real plane pitch
    static constexpr int SPP = F * V + 1;     // spectrum plane pitch (float2): channel-strided
                                              // accesses of a warp land on distinct banks
    static constexpr int BYTES_R = CB * PP * 4;
    static constexpr int BYTES_C = CB * SPP * 8;
    static constexpr int BYTES = BYTES_R > BYTES_C ? BYTES_R : BYTES_C;
};

// Forward: src tile (real) -> spectrum dst[bin][plane][c], bin = u * (F/2+1) + v.
template <int F>
__global__ void __launch_bounds__(256) fft_forward_kernel(const float* __restrict__ src, TileMap m,
                                                          float2* __restrict__ dst) {
    using Cf = FftCfg<F>;
    constexpr int CB = Cf::CB, V = Cf::V;
    __shared__ __align__(16) unsigned char smem[Cf::BYTES];
    float* re = reinterpret_cast<float*>(smem);
    float2* sp = reinterpret_cast<float2*>(smem);
    const int64_t plane = blockIdx.x;
    const int c0 = blockIdx.y * CB;
    const int n = (int)(plane / m.tiles), t = (int)(plane - (int64_t)n * m.tiles);
    const int ty = t / m.tiles_x, tx = t - ty * m.tiles_x;
    const int h0 = ty * m.Th + m.oh, w0 = tx * m.Tw + m.ow;
    // all loads of the tile in flight at once (registers), then the shared-memory stores
    constexpr int NL = CB * F * F / 256;
    float ld[NL];
#pragma unroll
    for (int l = 0; l < NL; ++l) {
        const int idx = threadIdx.x + l * 256;
        const int cc = idx % CB, pix = idx / CB, i = pix / F, j = pix - i * F;
        const int h = h0 + i, w = w0 + j, c = c0 + cc;
        ld[l] = 0.f;
        if (i < m.rh && j < m.rw && (unsigned)h < (unsigned)m.H && (unsigned)w < (unsigned)m.W && c < m.C)
            ld[l] = __ldg(src + (((int64_t)n * m.H + h) * m.W + w) * m.C + c);
    }
#pragma unroll
    for (int l = 0; l < NL; ++l) {
        const int idx = threadIdx.x + l * 256;
        const int cc = idx % CB, pix = idx / CB, i = pix / F, j = pix - i * F;
        re[cc * Cf::PP + i * Cf::RP + j] = ld[l];
    }
    __syncthreads();
    // rows: thread = (channel, row), real -> complex, keep bins v <= F/2
    const int cr = threadIdx.x / F, row = threadIdx.x % F;
    float2 z[F];
#pragma unroll
    for (int j = 0; j < F; ++j) z[j] = make_float2(re[cr * Cf::PP + row * Cf::RP + j], 0.f);
    dft<F, false>(z);
    __syncthreads();  // the real tile is dead: the spectrum aliases it
#pragma unroll
    for (int v = 0; v < V; ++v) sp[cr * Cf::SPP + row * V + v] = z[v];
    __syncthreads();
    // columns of the Hermitian half: thread = (channel, v)
    if (threadIdx.x < CB * V) {
        const int cc = threadIdx.x / V, v = threadIdx.x % V;
#pragma unroll
        for (int u = 0; u < F; ++u) z[u] = sp[cc * Cf::SPP + u * V + v];
        dft<F, false>(z);
#pragma unroll
        for (int u = 0; u < F; ++u) sp[cc * Cf::SPP + u * V + v] = z[u];
    }
    __syncthreads();
    for (int idx = threadIdx.x; idx < F * V * CB; idx += 256) {
        const int cc = idx % CB, bin = idx / CB, u = bin / V, v = bin - u * V;
        if (c0 + cc < m.C) dst[((int64_t)bin * m.planes + plane) * m.C + c0 + cc] = sp[cc * Cf::SPP + u * V + v];
    }
}

// Inverse: spectrum src[bin][plane][c] -> real tile, window (oh, ow) + [0, Th) x [0, Tw)
// written to the NHWC tensor at (ty*Th, tx*Tw): out = alpha * v + beta * out.
template <int F>
__global__ void __launch_bounds__(256) fft_inverse_kernel(const float2* __restrict__ src, TileMap m, float alpha,
                                                          float beta, float* dst) {
    using Cf = FftCfg<F>;
    constexpr int CB = Cf::CB, V = Cf::V;
    __shared__ __align__(16) unsigned char smem[Cf::BYTES];
    float* re = reinterpret_cast<float*>(smem);
    float2* sp = reinterpret_cast<float2*>(smem);
    const int64_t plane = blockIdx.x;
    const int c0 = blockIdx.y * CB;
    const int n = (int)(plane / m.tiles), t = (int)(plane - (int64_t)n * m.tiles);
    const int ty = t / m.tiles_x, tx = t - ty * m.tiles_x;
    constexpr int NL = (F * V * CB + 255) / 256;
    float2 ld[NL];
#pragma unroll
    for (int l = 0; l < NL; ++l) {
        const int idx = threadIdx.x + l * 256;
        const int cc = idx % CB, bin = idx / CB;
        ld[l] = make_float2(0.f, 0.f);
        if (idx < F * V * CB && c0 + cc < m.C) ld[l] = __ldg(src + ((int64_t)bin * m.planes + plane) * m.C + c0 + cc);
    }
#pragma unroll
    for (int l = 0; l < NL; ++l) {
        const int idx = threadIdx.x + l * 256;
        const int cc = idx % CB, bin = idx / CB, u = bin / V, v = bin - u * V;
        if (idx < F * V * CB) sp[cc * Cf::SPP + u * V + v] = ld[l];
    }
    __syncthreads();
    float2 z[F];
    if (threadIdx.x < CB * V) {
        const int cc = threadIdx.x / V, v = threadIdx.x % V;
#pragma unroll
        for (int u = 0; u < F; ++u) z[u] = sp[cc * Cf::SPP + u * V + v];
        dft<F, true>(z);
#pragma unroll
        for (int u = 0; u < F; ++u) sp[cc * Cf::SPP + u * V + v] = z[u];
    }
    __syncthreads();
    // rows: Hermitian half -> full spectrum -> real row
    const int cr = threadIdx.x / F, row = threadIdx.x % F;
#pragma unroll
    for (int v = 0; v < V; ++v) z[v] = sp[cr * Cf::SPP + row * V + v];
#pragma unroll
    for (int v = 1; v < F / 2; ++v) z[F - v] = make_float2(z[v].x, -z[v].y);
    dft<F, true>(z);
    __syncthreads();  // spectrum dead: the real tile aliases it
#pragma unroll
    for (int j = 0; j < F; ++j) re[cr * Cf::PP + row * Cf::RP + j] = z[j].x;
    __syncthreads();
    const int h0 = ty * m.Th, w0 = tx * m.Tw;
    for (int idx = threadIdx.x; idx < CB * m.Th * m.Tw; idx += 256) {
        const int cc = idx % CB, pix = idx / CB, i = pix / m.Tw, j = pix - i * m.Tw;
        const int h = h0 + i, w = w0 + j, c = c0 + cc;
        if (h >= m.H || w >= m.W || c >= m.C) continue;
        float* d = dst + (((int64_t)n * m.H + h) * m.W + w) * m.C + c;
        float v = alpha * re[cc * Cf::PP + (i + m.oh) * Cf::RP + j + m.ow];
        if (beta != 0.f) v += beta * *d;
        *d = v;
    }
}

// Per-bin complex GEMM C[z][m][n] = sum_k opA(m, k) * opB(n, k), z = bin (grid.z).
// KA: A(m, k) = A[m * lda + k] (else A[k * lda + m]); KB likewise for B(n, k);
// CJA / CJB conjugate the operand.  BM x 64 outputs per CTA (BM = 64, 32 or 16: few
// planes per bin at small micro-batches), 8 / 16 / 32 k per stage, 16 x 16 threads, each with
// TM = BM/16 rows and 4 columns in 2-wide blocks half a tile apart (conflict-free
// 16-byte shared-memory reads), register prefetch of the next stage.
template <int BM>
__device__ __forceinline__ int crow(int ty, int i) {
    if constexpr (BM == 64) return i < 2 ? ty * 2 + i : 32 + ty * 2 + i - 2;
    else if constexpr (BM == 32) return ty * 2 + i;
    else return ty;
}

template <int BM, bool KA, bool KB, bool CJA, bool CJB>
__global__ void __launch_bounds__(256, 2) cgemm_kernel(const float2* __restrict__ A, const float2* __restrict__ B,
                                                    float2* __restrict__ Cm, int M, int N, int K, int lda, int ldb,
                                                    int ldc, int64_t sA, int64_t sB, int64_t sC, int accum) {
    // deeper k stages for the short tiles: more bytes in flight when few planes make
    // the per-bin filter spectrum read the bound (BM * BK + 64 * BK complex per stage)
    constexpr int BN = 64, BK = BM == 16 ? 32 : BM == 32 ? 16 : 8, PAD = 4, TM = BM / 16;
    constexpr int NA = (BM * BK + 255) / 256, NB = BN * BK / 256;
    __shared__ __align__(16) float2 As[2][BK][BM + PAD];
    __shared__ __align__(16) float2 Bs[2][BK][BN + PAD];
    A += blockIdx.z * sA; B += blockIdx.z * sB; Cm += blockIdx.z * sC;
    const int m0 = blockIdx.x * BM, n0 = blockIdx.y * BN;
    const int t = threadIdx.x, tx = t % 16, ty = t / 16;
    // element e of a stage: k-contiguous operands walk k fastest, the others m / n
    auto a_coord = [&](int e, int& mm, int& kk) {
        if (KA) { mm = e / BK; kk = e % BK; } else { kk = e / BM; mm = e % BM; }
    };
    auto b_coord = [&](int e, int& nn, int& kk) {
        if (KB) { nn = e / BK; kk = e % BK; } else { kk = e / BN; nn = e % BN; }
    };
    float2 ra[NA], rb[NB];
    auto load = [&](int k0) {
#pragma unroll
        for (int i = 0; i < NA; ++i) {
            const int e = t + i * 256;
            int mm, kk;
            a_coord(e, mm, kk);
            float2 v = make_float2(0.f, 0.f);
            if (e < BM * BK && m0 + mm < M && k0 + kk < K)
                v = __ldg(KA ? A + (int64_t)(m0 + mm) * lda + k0 + kk : A + (int64_t)(k0 + kk) * lda + m0 + mm);
            if (CJA) v.y = -v.y;
            ra[i] = v;
        }
#pragma unroll
        for (int i = 0; i < NB; ++i) {
            const int e = t + i * 256;
            int nn, kk;
            b_coord(e, nn, kk);
            float2 u = make_float2(0.f, 0.f);
            if (n0 + nn < N && k0 + kk < K)
                u = __ldg(KB ? B + (int64_t)(n0 + nn) * ldb + k0 + kk : B + (int64_t)(k0 + kk) * ldb + n0 + nn);
            if (CJB) u.y = -u.y;
            rb[i] = u;
        }
    };
    auto store = [&](int buf) {
#pragma unroll
        for (int i = 0; i < NA; ++i) {
            const int e = t + i * 256;
            int mm, kk;
            a_coord(e, mm, kk);
            if (e < BM * BK) As[buf][kk][mm] = ra[i];
        }
#pragma unroll
        for (int i = 0; i < NB; ++i) {
            int nn, kk;
            b_coord(t + i * 256, nn, kk);
            Bs[buf][kk][nn] = rb[i];
        }
    };
    float2 acc[TM][4];
#pragma unroll
    for (int i = 0; i < TM; ++i)
#pragma unroll
        for (int j = 0; j < 4; ++j) acc[i][j] = make_float2(0.f, 0.f);
    load(0);
    store(0);
    __syncthreads();
    int buf = 0;
    for (int k0 = 0; k0 < K; k0 += BK) {
        const bool more = k0 + BK < K;
        if (more) load(k0 + BK);
#pragma unroll
        for (int k = 0; k < BK; ++k) {
            float2 a[TM], b[4];
            if constexpr (TM == 1) {
                a[0] = As[buf][k][ty];
            } else {
#pragma unroll
                for (int h = 0; h < TM / 2; ++h) {
                    const float4 av = *reinterpret_cast<const float4*>(&As[buf][k][crow<BM>(ty, 2 * h)]);
                    a[2 * h] = make_float2(av.x, av.y); a[2 * h + 1] = make_float2(av.z, av.w);
                }
            }
            const float4 b0 = *reinterpret_cast<const float4*>(&Bs[buf][k][tx * 2]);
            const float4 b1 = *reinterpret_cast<const float4*>(&Bs[buf][k][32 + tx * 2]);
            b[0] = make_float2(b0.x, b0.y); b[1] = make_float2(b0.z, b0.w);
            b[2] = make_float2(b1.x, b1.y); b[3] = make_float2(b1.z, b1.w);
#pragma unroll
            for (int i = 0; i < TM; ++i)
#pragma unroll
                for (int j = 0; j < 4; ++j) {
                    acc[i][j].x = fmaf(a[i].x, b[j].x, acc[i][j].x);
                    acc[i][j].x = fmaf(-a[i].y, b[j].y, acc[i][j].x);
                    acc[i][j].y = fmaf(a[i].x, b[j].y, acc[i][j].y);
                    acc[i][j].y = fmaf(a[i].y, b[j].x, acc[i][j].y);
                }
        }
        if (more) store(buf ^ 1);
        __syncthreads();
        buf ^= 1;
    }
#pragma unroll
    for (int i = 0; i < TM; ++i) {
        const int mm = m0 + crow<BM>(ty, i);
        if (mm >= M) continue;
#pragma unroll
        for (int j = 0; j < 4; ++j) {
            const int nn = n0 + (j < 2 ? tx * 2 + j : 32 + tx * 2 + j - 2);
            if (nn < N) {
                float2* d = Cm + (int64_t)mm * ldc + nn;
                if (accum) { const float2 o = *d; *d = make_float2(o.x + acc[i][j].x, o.y + acc[i][j].y); }
                else *d = acc[i][j];
            }
        }
    }
}

template <bool KA, bool KB, bool CJA, bool CJB>
int cgemm(const float2* A, const float2* B, float2* C, int M, int N, int K, int lda, int ldb, int ldc, int64_t sA,
          int64_t sB, int64_t sC, int64_t batch, cudaStream_t st, int accum = 0) {
    const int bm = M <= 16 ? 16 : M <= 32 ? 32 : 64;
    dim3 grid((unsigned)ceil_div(M, bm), (unsigned)ceil_div(N, 64), (unsigned)batch);
    if (bm == 16)
        cgemm_kernel<16, KA, KB, CJA, CJB><<<grid, 256, 0, st>>>(A, B, C, M, N, K, lda, ldb, ldc, sA, sB, sC, accum);
    else if (bm == 32)
        cgemm_kernel<32, KA, KB, CJA, CJB><<<grid, 256, 0, st>>>(A, B, C, M, N, K, lda, ldb, ldc, sA, sB, sC, accum);
    else
        cgemm_kernel<64, KA, KB, CJA, CJB><<<grid, 256, 0, st>>>(A, B, C, M, N, K, lda, ldb, ldc, sA, sB, sC, accum);
    count_launch();
    return (int)cudaGetLastError();
}

template <int F>
int fwd_t(const float* src, const TileMap& m, float2* dst, cudaStream_t st) {
    dim3 grid((unsigned)m.planes, (unsigned)ceil_div(m.C, FftCfg<F>::CB));
    fft_forward_kernel<F><<<grid, 256, 0, st>>>(src, m, dst);
    count_launch();
    return (int)cudaGetLastError();
}
template <int F>
int inv_t(const float2* src, const TileMap& m, float alpha, float beta, float* dst, cudaStream_t st) {
    dim3 grid((unsigned)m.planes, (unsigned)ceil_div(m.C, FftCfg<F>::CB));
    fft_inverse_kernel<F><<<grid, 256, 0, st>>>(src, m, alpha, beta, dst);
    count_launch();
    return (int)cudaGetLastError();
}
int fft_forward(int F, const float* src, const TileMap& m, float2* dst, cudaStream_t st) {
    switch (F) {
        case 8: return fwd_t<8>(src, m, dst, st);
        case 16: return fwd_t<16>(src, m, dst, st);
        case 32: return fwd_t<32>(src, m, dst, st);
    }
    return -1;
}
int fft_inverse(int F, const float2* src, const TileMap& m, float alpha, float beta, float* dst, cudaStream_t st) {
    switch (F) {
        case 8: return inv_t<8>(src, m, alpha, beta, dst, st);
        case 16: return inv_t<16>(src, m, alpha, beta, dst, st);
        case 32: return inv_t<32>(src, m, alpha, beta, dst, st);
    }
    return -1;
}

// Tile map of an operand over the grid of the transform's output tiles.
TileMap tile_map(const FftGeom& z, int H, int W, int C, int oh, int ow, int rh, int rw, int64_t planes) {
    return TileMap{H, W, C, z.tiles_x, z.tiles_y * z.tiles_x, z.Th, z.Tw, oh, ow, rh, rw, planes};
}

}  // namespace

bool fft_geom(const Geom& g, int type, int algo, FftGeom* z) {
    if (g.math != MUCU_MATH_F32 || g.stride != 1) return false;
    if (algo != MUCU_ALGO_FFT && algo != MUCU_ALGO_FFT_TILING) return false;
    const int Eh = type == MUCU_BWD_DATA ? g.h : g.p, Ew = type == MUCU_BWD_DATA ? g.w : g.q;
    if (Eh < 1 || Ew < 1) return false;
    if (algo == MUCU_ALGO_FFT) {
        const int need = std::max(Eh + g.r - 1, Ew + g.s - 1);
        int F = 8;
        while (F < need) F *= 2;
        if (F > 32) return false;
        z->F = F; z->Th = Eh; z->Tw = Ew;
    } else {
        if (g.r > 16 || g.s > 16) return false;
        z->F = 32;
        z->Th = std::min(Eh, 33 - g.r);
        z->Tw = std::min(Ew, 33 - g.s);
    }
    z->tiles_y = (int)ceil_div(Eh, z->Th);
    z->tiles_x = (int)ceil_div(Ew, z->Tw);
    z->bins = (int64_t)z->F * (z->F / 2 + 1);
    return true;
}

int fft_run(const Geom& g, int type, int algo, int32_t b, float alpha, const float* in0, const float* in1, float beta,
            float* out, char* ws, const WsLayout& L, CallCtx* ctx, cudaStream_t st) {
    FftGeom z;
    if (!fft_geom(g, type, algo, &z)) return -1;
    const int F = z.F;
    const int64_t planes = (int64_t)b * z.tiles_y * z.tiles_x, bins = z.bins;
    const float scale = alpha / (float)(F * F);
    float2* Wf = (float2*)(ws + L.fixed_off);
    float2* Sa = (float2*)(ws + L.a_off);
    float2* Sb = (float2*)(ws + L.b_off);
    int e = 0;
    if (type != MUCU_BWD_FILTER && (ctx->fixed_kind != 5 || ctx->fixed_src != in1)) {
        // filter spectrum [bin][k][c]: filters as K images of R x S pixels, C channels
        TileMap fm{g.r, g.s, g.c, 1, 1, g.r, g.s, 0, 0, g.r, g.s, g.k};
        e = fft_forward(F, in1, fm, Wf, st);
        if (e) return e;
        ctx->fixed_kind = 5;
        ctx->fixed_src = in1;
    }
    if (type == MUCU_FWD) {
        // X[bin][plane][c] of x tiles from (ty*Th - pad, tx*Tw - pad); Y = X . conj(W)
        e = fft_forward(F, in0, tile_map(z, g.h, g.w, g.c, -g.pad, -g.pad, F, F, planes), Sa, st);
        if (!e) e = cgemm<true, true, false, true>(Sa, Wf, Sb, (int)planes, g.k, g.c, g.c, g.c, g.k, planes * g.c,
                                                   (int64_t)g.k * g.c, planes * g.k, bins, st);
        if (!e) e = fft_inverse(F, Sb, tile_map(z, g.p, g.q, g.k, 0, 0, 0, 0, planes), scale, beta, out, st);
    } else if (type == MUCU_BWD_DATA) {
        // DY tiles from (ty*Th + pad - (R-1), ...); DX = DY . W, window from (R-1, S-1)
        e = fft_forward(F, in0,
                        tile_map(z, g.p, g.q, g.k, g.pad - (g.r - 1), g.pad - (g.s - 1), F, F, planes), Sa, st);
        if (!e) e = cgemm<true, false, false, false>(Sa, Wf, Sb, (int)planes, g.c, g.k, g.k, g.c, g.c, planes * g.k,
                                                     (int64_t)g.k * g.c, planes * g.c, bins, st);
        if (!e) e = fft_inverse(F, Sb, tile_map(z, g.h, g.w, g.c, g.r - 1, g.s - 1, 0, 0, planes), scale, beta, out, st);
    } else {
        // X tiles as FWD; DY zero outside its own tile; DW[bin][k][c] = sum_planes conj(DY) X.
        // Consecutive micro-batches of this algorithm accumulate DW in the frequency domain
        // (the transform is linear: sum_mb IFFT(S_mb) = IFFT(sum_mb S_mb)) and the inverse
        // runs once, at the last of them, with the first one's beta (P:L58 output scale).
        float2* DW = (float2*)(ws + L.fixed_off);
        const bool first = ctx->fixed_kind != 6;
        if (first) { ctx->fixed_kind = 6; ctx->fixed_src = nullptr; ctx->fft_beta = beta; }
        e = fft_forward(F, in0, tile_map(z, g.h, g.w, g.c, -g.pad, -g.pad, F, F, planes), Sa, st);
        if (!e) e = fft_forward(F, in1, tile_map(z, g.p, g.q, g.k, 0, 0, z.Th, z.Tw, planes), Sb, st);
        if (!e) e = cgemm<false, false, true, false>(Sb, Sa, DW, g.k, g.c, (int)planes, g.k, g.c, g.c, planes * g.k,
                                                     planes * g.c, (int64_t)g.k * g.c, bins, st, first ? 0 : 1);
        // dw[k][r][s][c]: K "images" of R x S, window at the origin
        TileMap om{g.r, g.s, g.c, 1, 1, g.r, g.s, 0, 0, 0, 0, g.k};
        if (!e && ctx->next_algo != algo) {
            e = fft_inverse(F, DW, om, scale, ctx->fft_beta, out, st);
            ctx->fixed_kind = 0;
        }
    }
    return e;
}

}  // namespace mucu
