// kernels_elem.cu -- data-movement kernels of the workspace-using algorithms.
//
//   im2col            (algorithm (b), "explicit GEMM"): x -> col[b*P*Q][kpitch]
//   pad_filter        KRSC filter copied to a 16-B aligned row pitch (for TMA)
//   col2im            deterministic gather-sum dcol -> dx (no atomics)
//   wg_filter/input/output   Winograd F(2x2,3x3) transforms (algorithm (c),
//                     Lavin & Gray, PAPER.md ref [23] P:L317)
//
// These passes are HBM-bound (no reuse beyond a few neighbouring pixels):
// grid-stride loops with the channel index fastest so that consecutive threads
// touch consecutive addresses (coalesced), 16-byte vectors where C allows,
// grid sized to a multiple of the SM count.
#include <cuda_bf16.h>
#include <cuda_runtime.h>

#include <type_traits>

#include "mucudnn_internal.h"

namespace mucu {

// Programmatic dependent launch (see kernels_tc.cu launch_t): every kernel here
// is launched with programmatic stream serialization and waits for the
// previous kernel's results before its first global access, so its launch
// and scheduling overlap the previous kernel's tail.
__device__ __forceinline__ void pdl_entry() {
    asm volatile("griddepcontrol.wait;" ::: "memory");
    asm volatile("griddepcontrol.launch_dependents;" :::);
}

// (FastDiv, mucudnn_internal.h: division by a runtime divisor d >= 1 as a
// multiply-high, l = ceil(log2 d), m = floor(2^32 (2^l - d) / d) + 1, exact for all
// 32-bit n -- the index math of the memory-bound transform kernels below was
// dominated by integer divisions.)
template <typename... KArgs, typename... Args>
void launch_pdl(void (*kern)(KArgs...), dim3 grid, dim3 block, size_t smem, cudaStream_t st, Args... args) {
    static const int pdl = getenv("MUCU_PDL") ? atoi(getenv("MUCU_PDL")) : 1;
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = grid;
    cfg.blockDim = block;
    cfg.dynamicSmemBytes = smem;
    cfg.stream = st;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = attr;
    cfg.numAttrs = pdl ? 1 : 0;
    cudaLaunchKernelEx(&cfg, kern, ((KArgs)args)...);
}


namespace {

template <class T> __device__ __forceinline__ float to_f(T v);
template <> __device__ __forceinline__ float to_f<float>(float v) { return v; }
template <> __device__ __forceinline__ float to_f<__nv_bfloat16>(__nv_bfloat16 v) { return __bfloat162float(v); }
template <class T> __device__ __forceinline__ T from_f(float v);
template <> __device__ __forceinline__ float from_f<float>(float v) { return v; }
template <> __device__ __forceinline__ __nv_bfloat16 from_f<__nv_bfloat16>(float v) { return __float2bfloat16_rn(v); }

int grid_for(int64_t work, int threads) {
    int dev = 0, sms = 148;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    int64_t blocks = (work + threads - 1) / threads;
    int64_t cap = (int64_t)sms * 16;
    if (blocks > cap) blocks = cap;
    if (blocks < 1) blocks = 1;
    return (int)blocks;
}

template <class T>
__global__ void pad_filter_kernel(const T* __restrict__ w, T* __restrict__ wp, int K, int RSC, int kpitch) {
    pdl_entry();
    const int64_t total = (int64_t)K * kpitch;
    for (int64_t idx = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; idx < total;
         idx += (int64_t)gridDim.x * blockDim.x) {
        int k = (int)(idx / kpitch), kk = (int)(idx % kpitch);
        wp[idx] = kk < RSC ? w[(int64_t)k * RSC + kk] : from_f<T>(0.f);
    }
}

// ------------------------------------------------------------- Winograd --
// F(2x2,3x3) (Lavin & Gray, ref [23]):
//   G  = [[1,0,0],[1/2,1/2,1/2],[1/2,-1/2,1/2],[0,0,1]]
//   B^T= [[1,0,-1,0],[0,1,1,0],[0,-1,1,0],[0,1,0,-1]]
//   A^T= [[1,1,1,0],[0,1,-1,-1]]
// Y = A^T [ (G g G^T) .* (B^T d B) ] A, per 4x4 input tile (tile stride 2).
// Layouts: U[xi][o][i], V[xi][t][i], M[xi][t][o] with xi = 4*a + b, o = output
// channel, i = input channel, t = (n, tile_h, tile_w).
// FWD: i = C, o = K, g = w[o,:,:,i].  DGRAD (full conv with the 180-degree
// rotated, C/K-swapped filter; pad' = 2 - pad): i = K, o = C,
// g[r][s] = w[i, 2-r, 2-s, o].
template <class T>
__global__ void wg_filter_kernel(const T* __restrict__ w, T* __restrict__ U, int O, int I, int C, bool dgrad) {
    pdl_entry();
    const int64_t total = (int64_t)O * I;
    for (int64_t idx = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; idx < total;
         idx += (int64_t)gridDim.x * blockDim.x) {
        int i = (int)(idx % I), o = (int)(idx / I);
        float g[3][3];
        for (int r = 0; r < 3; ++r)
            for (int s = 0; s < 3; ++s) {
                // w is KRSC: element (k, r, s, c)
                g[r][s] = dgrad ? to_f<T>(w[(((int64_t)i * 3 + (2 - r)) * 3 + (2 - s)) * C + o])
                                : to_f<T>(w[(((int64_t)o * 3 + r) * 3 + s) * C + i]);
            }
        float t[4][3];  // t = G g
        for (int s = 0; s < 3; ++s) {
            t[0][s] = g[0][s];
            t[1][s] = 0.5f * (g[0][s] + g[1][s] + g[2][s]);
            t[2][s] = 0.5f * (g[0][s] - g[1][s] + g[2][s]);
            t[3][s] = g[2][s];
        }
        for (int a = 0; a < 4; ++a) {  // u = t G^T
            float u0 = t[a][0];
            float u1 = 0.5f * (t[a][0] + t[a][1] + t[a][2]);
            float u2 = 0.5f * (t[a][0] - t[a][1] + t[a][2]);
            float u3 = t[a][2];
            const int64_t plane = (int64_t)O * I;
            U[(a * 4 + 0) * plane + idx] = from_f<T>(u0);
            U[(a * 4 + 1) * plane + idx] = from_f<T>(u1);
            U[(a * 4 + 2) * plane + idx] = from_f<T>(u2);
            U[(a * 4 + 3) * plane + idx] = from_f<T>(u3);
        }
    }
}

// V[xi][t][i] = (B^T d B)[xi], d = 4x4 patch of `in` ([b, IH, IW, I]) at
// (2*th - pad, 2*tw - pad), zero outside.  TH x TW tiles per image.
template <class T>
__global__ void wg_input_kernel(const T* __restrict__ in, T* __restrict__ V, int64_t tiles, int IH, int IW,
                                int I, int TH, int TW, int pad) {
    pdl_entry();
    const int64_t total = tiles * I;
    for (int64_t idx = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; idx < total;
         idx += (int64_t)gridDim.x * blockDim.x) {
        int i = (int)(idx % I);
        int64_t t = idx / I;
        int tw = (int)(t % TW);
        int64_t t2 = t / TW;
        int th = (int)(t2 % TH);
        int n = (int)(t2 / TH);
        float d[4][4];
        for (int a = 0; a < 4; ++a)
            for (int b = 0; b < 4; ++b) {
                int h = 2 * th - pad + a, w = 2 * tw - pad + b;
                d[a][b] = (h >= 0 && h < IH && w >= 0 && w < IW)
                              ? to_f<T>(in[(((int64_t)n * IH + h) * IW + w) * I + i]) : 0.f;
            }
        float e[4][4];  // e = B^T d
        for (int b = 0; b < 4; ++b) {
            e[0][b] = d[0][b] - d[2][b];
            e[1][b] = d[1][b] + d[2][b];
            e[2][b] = d[2][b] - d[1][b];
            e[3][b] = d[1][b] - d[3][b];
        }
        const int64_t plane = tiles * I;
        for (int a = 0; a < 4; ++a) {  // v = e B
            float v0 = e[a][0] - e[a][2];
            float v1 = e[a][1] + e[a][2];
            float v2 = e[a][2] - e[a][1];
            float v3 = e[a][1] - e[a][3];
            V[(a * 4 + 0) * plane + idx] = from_f<T>(v0);
            V[(a * 4 + 1) * plane + idx] = from_f<T>(v1);
            V[(a * 4 + 2) * plane + idx] = from_f<T>(v2);
            V[(a * 4 + 3) * plane + idx] = from_f<T>(v3);
        }
    }
}

// 4 consecutive channels as one 16-B (fp32) / 8-B (bf16) access.
__device__ __forceinline__ void ld4(const float* p, float (&o)[4]) {
    const float4 v = __ldg(reinterpret_cast<const float4*>(p));
    o[0] = v.x; o[1] = v.y; o[2] = v.z; o[3] = v.w;
}
__device__ __forceinline__ void ld4(const __nv_bfloat16* p, float (&o)[4]) {
    const uint2 u = __ldg(reinterpret_cast<const uint2*>(p));
    const __nv_bfloat162 a = *reinterpret_cast<const __nv_bfloat162*>(&u.x), b = *reinterpret_cast<const __nv_bfloat162*>(&u.y);
    o[0] = __low2float(a); o[1] = __high2float(a); o[2] = __low2float(b); o[3] = __high2float(b);
}
__device__ __forceinline__ void st4(float* p, const float (&v)[4]) {
    *reinterpret_cast<float4*>(p) = make_float4(v[0], v[1], v[2], v[3]);
}
__device__ __forceinline__ void st4(__nv_bfloat16* p, const float (&v)[4]) {
    uint2 u;
    *reinterpret_cast<__nv_bfloat162*>(&u.x) = __floats2bfloat162_rn(v[0], v[1]);
    *reinterpret_cast<__nv_bfloat162*>(&u.y) = __floats2bfloat162_rn(v[2], v[3]);
    *reinterpret_cast<uint2*>(p) = u;
}

// wg_input_kernel / wgw_x_kernel, 4 channels per thread (I % 4 == 0): vector loads /
// stores, tile index by multiply-high division.  Same arithmetic per channel
// (bit-identical V).  Rows t of pitch Ip (>= I channels; padding channels and rows
// t >= tiles are zero), planes of `plane` elements.
template <class T>
__global__ void wg_input4_kernel(const T* __restrict__ in, T* __restrict__ V, uint32_t total, int IH, int IW, int I,
                                 int Ip, uint32_t tiles, FastDiv dI4, FastDiv dTW, FastDiv dTH, int pad,
                                 int64_t plane) {
    pdl_entry();
    for (uint32_t idx = blockIdx.x * blockDim.x + threadIdx.x; idx < total; idx += gridDim.x * blockDim.x) {
        const uint32_t t = dI4.div(idx), i = 4 * (idx - t * dI4.d);
        const uint32_t t2 = dTW.div(t), tw = t - t2 * dTW.d;
        const uint32_t n = dTH.div(t2), th = t2 - n * dTH.d;
        const bool live = t < tiles && (int)i < I;
        float d[4][4][4];
#pragma unroll
        for (int a = 0; a < 4; ++a)
#pragma unroll
            for (int b = 0; b < 4; ++b) {
                const int h = 2 * (int)th - pad + a, w = 2 * (int)tw - pad + b;
                if (live && h >= 0 && h < IH && w >= 0 && w < IW) {
                    ld4(in + (((int64_t)n * IH + h) * IW + w) * I + i, d[a][b]);
                } else {
#pragma unroll
                    for (int u = 0; u < 4; ++u) d[a][b][u] = 0.f;
                }
            }
        T* out = V + (int64_t)t * Ip + i;
#pragma unroll
        for (int a = 0; a < 4; ++a) {
            float e0[4], e1[4], e2[4], e3[4];  // row a of e = B^T d, per channel
#pragma unroll
            for (int b = 0; b < 4; ++b)
#pragma unroll
                for (int u = 0; u < 4; ++u) {
                    const float v = a == 0 ? d[0][b][u] - d[2][b][u]
                                  : a == 1 ? d[1][b][u] + d[2][b][u]
                                  : a == 2 ? d[2][b][u] - d[1][b][u]
                                           : d[1][b][u] - d[3][b][u];
                    (b == 0 ? e0 : b == 1 ? e1 : b == 2 ? e2 : e3)[u] = v;
                }
            float v0[4], v1[4], v2[4], v3[4];  // v = e B
#pragma unroll
            for (int u = 0; u < 4; ++u) {
                v0[u] = e0[u] - e2[u];
                v1[u] = e1[u] + e2[u];
                v2[u] = e2[u] - e1[u];
                v3[u] = e1[u] - e3[u];
            }
            st4(out + (a * 4 + 0) * plane, v0);
            st4(out + (a * 4 + 1) * plane, v1);
            st4(out + (a * 4 + 2) * plane, v2);
            st4(out + (a * 4 + 3) * plane, v3);
        }
    }
}

// wg_output_kernel, 4 channels per thread (O % 4 == 0).  Same arithmetic per channel.
template <class T>
__global__ void wg_output4_kernel(const float* __restrict__ M, T* __restrict__ out, uint32_t total, int OH, int OW,
                                  int O, FastDiv dO4, FastDiv dTW, FastDiv dTH, float alpha, float beta,
                                  int64_t plane) {
    pdl_entry();
    for (uint32_t idx = blockIdx.x * blockDim.x + threadIdx.x; idx < total; idx += gridDim.x * blockDim.x) {
        const uint32_t t = dO4.div(idx), o = 4 * (idx - t * dO4.d);
        const uint32_t t2 = dTW.div(t), tw = t - t2 * dTW.d;
        const uint32_t n = dTH.div(t2), th = t2 - n * dTH.d;
        const float* src = M + (int64_t)t * O + o;
        float z[2][4][4];  // z = A^T m, per channel
#pragma unroll
        for (int b = 0; b < 4; ++b) {
            float m0[4], m1[4], m2[4], m3[4];
            ld4(src + (0 * 4 + b) * plane, m0);
            ld4(src + (1 * 4 + b) * plane, m1);
            ld4(src + (2 * 4 + b) * plane, m2);
            ld4(src + (3 * 4 + b) * plane, m3);
#pragma unroll
            for (int u = 0; u < 4; ++u) {
                z[0][b][u] = m0[u] + m1[u] + m2[u];
                z[1][b][u] = m1[u] - m2[u] - m3[u];
            }
        }
#pragma unroll
        for (int a = 0; a < 2; ++a) {
            const int h = 2 * (int)th + a;
            if (h >= OH) continue;
#pragma unroll
            for (int j = 0; j < 2; ++j) {
                const int w = 2 * (int)tw + j;
                if (w >= OW) continue;
                T* dst = out + (((int64_t)n * OH + h) * OW + w) * O + o;
                float old[4] = {0.f, 0.f, 0.f, 0.f};
                if (beta != 0.f) ld4(dst, old);
                float y[4];
#pragma unroll
                for (int u = 0; u < 4; ++u) {
                    const float yv = j == 0 ? z[a][0][u] + z[a][1][u] + z[a][2][u] : z[a][1][u] - z[a][2][u] - z[a][3][u];
                    float v = alpha * yv;
                    if (beta != 0.f) v += beta * old[u];
                    y[u] = v;
                }
                st4(dst, y);
            }
        }
    }
}

// out[n, 2th+i, 2tw+j, o] = alpha * (A^T M A)[i][j] + beta * out (masked at the
// ragged right/bottom edge).
template <class T>
__global__ void wg_output_kernel(const float* __restrict__ M, T* __restrict__ out, int64_t tiles, int OH, int OW,
                                 int O, int TH, int TW, float alpha, float beta) {
    pdl_entry();
    const int64_t total = tiles * O;
    const int64_t plane = total;
    for (int64_t idx = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; idx < total;
         idx += (int64_t)gridDim.x * blockDim.x) {
        int o = (int)(idx % O);
        int64_t t = idx / O;
        int tw = (int)(t % TW);
        int64_t t2 = t / TW;
        int th = (int)(t2 % TH);
        int n = (int)(t2 / TH);
        float m[4][4];
        for (int a = 0; a < 4; ++a)
            for (int b = 0; b < 4; ++b) m[a][b] = M[(a * 4 + b) * plane + idx];
        float z[2][4];  // z = A^T m
        for (int b = 0; b < 4; ++b) {
            z[0][b] = m[0][b] + m[1][b] + m[2][b];
            z[1][b] = m[1][b] - m[2][b] - m[3][b];
        }
        for (int a = 0; a < 2; ++a) {
            float y0 = z[a][0] + z[a][1] + z[a][2];
            float y1 = z[a][1] - z[a][2] - z[a][3];
            int h = 2 * th + a;
            if (h >= OH) continue;
            for (int j = 0; j < 2; ++j) {
                int w = 2 * tw + j;
                if (w >= OW) continue;
                int64_t off = (((int64_t)n * OH + h) * OW + w) * O + o;
                float v = alpha * (j == 0 ? y0 : y1);
                if (beta != 0.f) v += beta * to_f<T>(out[off]);
                out[off] = from_f<T>(v);
            }
        }
    }
}

// Winograd F(3x3,2x2) BackwardFilter: per 2x2 tile of dy at
// (2th, 2tw) and the 4x4 x patch at (2th - pad, 2tw - pad),
//   dW[r][s] += (G^T [(A dy A^T) .* (B^T x B)] G)[r][s],
// A = [[1,0],[1,1],[1,-1],[0,-1]] (the transpose of F(2x2,3x3)'s A^T), B^T and G
// as in F(2x2,3x3).  V[xi][t][c] = (B^T x B)[xi], D[xi][t][k] = (A dy A^T)[xi];
// rows t in [tiles, Tp) are zero so the GEMMs can read whole k-blocks.
template <class T>
__global__ void wgw_x_kernel(const T* __restrict__ x, T* __restrict__ V, int64_t tiles, int64_t Tp, int H, int W,
                             int C, int Cp, int TH, int TW, int pad) {
    pdl_entry();
    const int64_t total = Tp * Cp, plane = Tp * Cp;
    for (int64_t idx = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; idx < total;
         idx += (int64_t)gridDim.x * blockDim.x) {
        const int c = (int)(idx % Cp);
        const int64_t t = idx / Cp;
        float d[4][4];
        if (t < tiles && c < C) {
            const int tw = (int)(t % TW);
            const int64_t t2 = t / TW;
            const int th = (int)(t2 % TH), n = (int)(t2 / TH);
            for (int a = 0; a < 4; ++a)
                for (int b = 0; b < 4; ++b) {
                    const int h = 2 * th - pad + a, w = 2 * tw - pad + b;
                    d[a][b] = (h >= 0 && h < H && w >= 0 && w < W) ? to_f<T>(x[(((int64_t)n * H + h) * W + w) * C + c])
                                                                   : 0.f;
                }
        } else {
            for (int a = 0; a < 4; ++a)
                for (int b = 0; b < 4; ++b) d[a][b] = 0.f;
        }
        float e[4][4];  // e = B^T d
        for (int b = 0; b < 4; ++b) {
            e[0][b] = d[0][b] - d[2][b];
            e[1][b] = d[1][b] + d[2][b];
            e[2][b] = d[2][b] - d[1][b];
            e[3][b] = d[1][b] - d[3][b];
        }
        for (int a = 0; a < 4; ++a) {  // v = e B
            V[(a * 4 + 0) * plane + idx] = from_f<T>(e[a][0] - e[a][2]);
            V[(a * 4 + 1) * plane + idx] = from_f<T>(e[a][1] + e[a][2]);
            V[(a * 4 + 2) * plane + idx] = from_f<T>(e[a][2] - e[a][1]);
            V[(a * 4 + 3) * plane + idx] = from_f<T>(e[a][1] - e[a][3]);
        }
    }
}

template <class T>
__global__ void wgw_dy_kernel(const T* __restrict__ dy, T* __restrict__ D, int64_t tiles, int64_t Tp, int P, int Q,
                              int K, int Kp, int TH, int TW) {
    pdl_entry();
    const int64_t total = Tp * Kp, plane = Tp * Kp;
    for (int64_t idx = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; idx < total;
         idx += (int64_t)gridDim.x * blockDim.x) {
        const int k = (int)(idx % Kp);
        const int64_t t = idx / Kp;
        float g[2][2] = {{0.f, 0.f}, {0.f, 0.f}};
        if (t < tiles && k < K) {
            const int tw = (int)(t % TW);
            const int64_t t2 = t / TW;
            const int th = (int)(t2 % TH), n = (int)(t2 / TH);
            for (int j = 0; j < 2; ++j)
                for (int l = 0; l < 2; ++l) {
                    const int p = 2 * th + j, q = 2 * tw + l;
                    if (p < P && q < Q) g[j][l] = to_f<T>(dy[(((int64_t)n * P + p) * Q + q) * K + k]);
                }
        }
        float e[4][2];  // e = A g
        for (int l = 0; l < 2; ++l) {
            e[0][l] = g[0][l];
            e[1][l] = g[0][l] + g[1][l];
            e[2][l] = g[0][l] - g[1][l];
            e[3][l] = -g[1][l];
        }
        for (int a = 0; a < 4; ++a) {  // (A g) A^T
            D[(a * 4 + 0) * plane + idx] = from_f<T>(e[a][0]);
            D[(a * 4 + 1) * plane + idx] = from_f<T>(e[a][0] + e[a][1]);
            D[(a * 4 + 2) * plane + idx] = from_f<T>(e[a][0] - e[a][1]);
            D[(a * 4 + 3) * plane + idx] = from_f<T>(-e[a][1]);
        }
    }
}

// dw[k][r][s][c] = alpha * (G^T M[.][k][c] G)[r][s] + beta * dw (beta = 0: no read).
__global__ void wgw_out_kernel(const float* __restrict__ M, float* __restrict__ dw, int K, int C, int Kp, int Cp,
                               float alpha, float beta) {
    pdl_entry();
    const int64_t total = (int64_t)K * C, plane = (int64_t)Kp * Cp;
    for (int64_t idx = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; idx < total;
         idx += (int64_t)gridDim.x * blockDim.x) {
        const int c = (int)(idx % C), k = (int)(idx / C);
        const int64_t mi = (int64_t)k * Cp + c;
        float m[4][4];
        for (int a = 0; a < 4; ++a)
            for (int b = 0; b < 4; ++b) m[a][b] = M[(a * 4 + b) * plane + mi];
        float z[3][4];  // z = G^T m
        for (int b = 0; b < 4; ++b) {
            z[0][b] = m[0][b] + 0.5f * (m[1][b] + m[2][b]);
            z[1][b] = 0.5f * (m[1][b] - m[2][b]);
            z[2][b] = 0.5f * (m[1][b] + m[2][b]) + m[3][b];
        }
        for (int r = 0; r < 3; ++r) {  // z G
            const float o[3] = {z[r][0] + 0.5f * (z[r][1] + z[r][2]), 0.5f * (z[r][1] - z[r][2]),
                                0.5f * (z[r][1] + z[r][2]) + z[r][3]};
            for (int s2 = 0; s2 < 3; ++s2) {
                float* d = dw + (((int64_t)k * 3 + r) * 3 + s2) * C + c;
                float v = alpha * o[s2];
                if (beta != 0.f) v += beta * *d;
                *d = v;
            }
        }
    }
}

// Row-oriented im2col: one warp per col row (output pixel m = (n,p,q)).  For
// a fixed filter row r the S*C values (s,c) of the row are CONTIGUOUS in NHWC
// x (x[n, h0+r, w0 .. w0+S-1, 0..C-1]), so the warp copies R runs of S*C
// elements with the lanes along the run (coalesced reads and writes, V-wide
// vectors when C % V == 0) and zero-fills outside [s_lo*C, s_hi*C) and rows
// off the image -- no per-element index division.
template <class T, int V>
__global__ void im2col_rows_kernel(const T* __restrict__ x, T* __restrict__ col, int64_t rows, int H, int W,
                                   int C, int P, int Q, int R, int S, int pad, int st, int kpitch) {
    pdl_entry();
    using VT = typename std::conditional<V == 1, T, uint4>::type;
    const int lane = threadIdx.x & 31;
    const int64_t warp0 = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    const int SC = S * C, RSC = R * SC;
    const int pq = P * Q;
    for (int64_t m = warp0; m < rows; m += nwarps) {
        const int n = (int)(m / pq);
        const int rem = (int)(m - (int64_t)n * pq);
        const int p = rem / Q, q = rem - (rem / Q) * Q;
        const int h0 = p * st - pad, w0 = q * st - pad;
        const int lo = max(0, -w0) * C, hi = min(S, W - w0) * C;
        T* dst = col + m * kpitch;
        for (int r = 0; r < R; ++r) {
            const int h = h0 + r;
            const bool hv = h >= 0 && h < H;
            const T* src = x + (((int64_t)n * H + (hv ? h : 0)) * W + w0) * C;  // may point left of the row; only read in [lo,hi)
            for (int sc = lane * V; sc < SC; sc += 32 * V) {
                VT v;
                if (hv && sc >= lo && sc < hi) v = *reinterpret_cast<const VT*>(src + sc);
                else if constexpr (V == 1) v = from_f<T>(0.f);
                else v = make_uint4(0, 0, 0, 0);
                *reinterpret_cast<VT*>(dst + r * SC + sc) = v;
            }
        }
        for (int kk = RSC + lane; kk < kpitch; kk += 32) dst[kk] = from_f<T>(0.f);
    }
}

// Small-C im2col (C not a multiple of the vector width, e.g. the RGB first
// layer): one thread per 16-byte chunk of a col row, so every store is a full
// coalesced 16-B vector; the chunk's V elements are gathered walking (r, s*C+c)
// incrementally from one division (reads hit L1/L2: neighbouring chunks share
// the same input rows).
template <class T>
__global__ void im2col_chunk_kernel(const T* __restrict__ x, T* __restrict__ col, int64_t rows, int H, int W,
                                    int C, int P, int Q, int R, int S, int pad, int st, int kpitch) {
    pdl_entry();
    constexpr int V = 16 / sizeof(T);
    const int SC = S * C, RSC = R * SC;
    const int cpr = kpitch / V;
    const int64_t total = rows * cpr;
    const int pq = P * Q;
    for (int64_t idx = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; idx < total;
         idx += (int64_t)gridDim.x * blockDim.x) {
        const int64_t m = idx / cpr;
        const int kk0 = (int)(idx - m * cpr) * V;
        const int n = (int)(m / pq);
        const int rem = (int)(m - (int64_t)n * pq);
        const int p = rem / Q, q = rem - (rem / Q) * Q;
        const int h0 = p * st - pad, w0 = q * st - pad;
        const int lo = max(0, -w0) * C, hi = min(S, W - w0) * C;
        int r = kk0 / SC, sc = kk0 - r * SC;
        const T* xn = x + (int64_t)n * H * W * C + (int64_t)w0 * C;
        __align__(16) T v[V];
#pragma unroll
        for (int e = 0; e < V; ++e) {
            T val = from_f<T>(0.f);
            const int h = h0 + r;
            if (r < R && sc >= lo && sc < hi && h >= 0 && h < H) val = xn[(int64_t)h * W * C + sc];
            v[e] = val;
            if (++sc == SC) { sc = 0; ++r; }
        }
        *reinterpret_cast<uint4*>(col + m * kpitch + kk0) = *reinterpret_cast<const uint4*>(v);
        (void)RSC;
    }
}

template <class T>
int im2col_t(const Geom& g, int32_t b, const void* x, void* col, int32_t kpitch, cudaStream_t st) {
    constexpr int V = 16 / sizeof(T);
    const int64_t rows = (int64_t)b * g.p * g.q;
    if (g.c % V == 0 && kpitch % V == 0) {
        const int grid = grid_for(rows * 32, 256);
        launch_pdl(im2col_rows_kernel<T, V>, dim3(grid), dim3(256), (size_t)(0), st, (const T*)x, (T*)col, rows, g.h, g.w, g.c, g.p, g.q, g.r,
                                                        g.s, g.pad, g.stride, kpitch);
    } else if (kpitch % V == 0) {
        const int grid = grid_for(rows * (kpitch / V), 256);
        launch_pdl(im2col_chunk_kernel<T>, dim3(grid), dim3(256), (size_t)(0), st, (const T*)x, (T*)col, rows, g.h, g.w, g.c, g.p, g.q, g.r,
                                                      g.s, g.pad, g.stride, kpitch);
    } else {
        const int grid = grid_for(rows * 32, 256);
        launch_pdl(im2col_rows_kernel<T, 1>, dim3(grid), dim3(256), (size_t)(0), st, (const T*)x, (T*)col, rows, g.h, g.w, g.c, g.p, g.q, g.r,
                                                        g.s, g.pad, g.stride, kpitch);
    }
    count_launch();
    return (int)cudaGetLastError();
}

template <class T>
__global__ void col2im_pixel_kernel(const float* __restrict__ dcol, T* __restrict__ dx, int64_t pixels, int H,
                                    int W, int C, int P, int Q, int R, int S, int pad, int st, int kpitch,
                                    float alpha, float beta) {
    pdl_entry();
    for (int64_t pix = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; pix < pixels;
         pix += (int64_t)gridDim.x * blockDim.x) {
        const int w = (int)(pix % W);
        const int64_t t2 = pix / W;
        const int h = (int)(t2 % H);
        const int n = (int)(t2 / H);
        const int hp = h + pad, wp = w + pad;
        const int r0 = hp % st, s0 = wp % st;
        float acc[4] = {0.f, 0.f, 0.f, 0.f};
        for (int r = r0, p = (hp - r0) / st; r < R && p >= 0; r += st, --p) {
            if (p >= P) continue;
            const float* rowp = dcol + ((int64_t)n * P + p) * Q * (int64_t)kpitch;
            for (int s = s0, q = (wp - s0) / st; s < S && q >= 0; s += st, --q) {
                if (q >= Q) continue;
                const float* src = rowp + (int64_t)q * kpitch + (r * S + s) * C;
                for (int c = 0; c < C; ++c) acc[c] += src[c];
            }
        }
        T* out = dx + pix * C;
        for (int c = 0; c < C; ++c) {
            float o = alpha * acc[c];
            if (beta != 0.f) o += beta * to_f<T>(out[c]);
            out[c] = from_f<T>(o);
        }
    }
}

// Gather col2im over the VALID taps only: for a dx pixel (h,w) the taps with
// st | h+pad-r are r = r0, r0+st, ... with r0 = (h+pad) % st, and p steps down
// by one per tap -- one division per pixel instead of two per tap.  One
// thread per (pixel, channel group of V channels), channels fastest.
template <class T, int V>
__global__ void col2im_taps_kernel(const float* __restrict__ dcol, T* __restrict__ dx, int64_t pixels, int H,
                                   int W, int C, int P, int Q, int R, int S, int pad, int st, int kpitch,
                                   float alpha, float beta) {
    pdl_entry();
    const int CG = C / V;
    const int64_t total = pixels * CG;
    for (int64_t idx = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; idx < total;
         idx += (int64_t)gridDim.x * blockDim.x) {
        const int c0 = (int)(idx % CG) * V;
        const int64_t pix = idx / CG;
        const int w = (int)(pix % W);
        const int64_t t2 = pix / W;
        const int h = (int)(t2 % H);
        const int n = (int)(t2 / H);
        const int hp = h + pad, wp = w + pad;
        const int r0 = hp % st, s0 = wp % st;
        float acc[V];
#pragma unroll
        for (int v = 0; v < V; ++v) acc[v] = 0.f;
        for (int r = r0, p = (hp - r0) / st; r < R && p >= 0; r += st, --p) {
            if (p >= P) continue;
            const float* rowp = dcol + ((int64_t)n * P + p) * Q * (int64_t)kpitch;
            for (int s = s0, q = (wp - s0) / st; s < S && q >= 0; s += st, --q) {
                if (q >= Q) continue;
                const float* src = rowp + (int64_t)q * kpitch + (r * S + s) * C + c0;
                if constexpr (V == 4) {
                    const float4 f = *reinterpret_cast<const float4*>(src);
                    acc[0] += f.x; acc[1] += f.y; acc[2] += f.z; acc[3] += f.w;
                } else {
#pragma unroll
                    for (int v = 0; v < V; ++v) acc[v] += src[v];
                }
            }
        }
        T* out = dx + pix * C + c0;
#pragma unroll
        for (int v = 0; v < V; ++v) {
            float o = alpha * acc[v];
            if (beta != 0.f) o += beta * to_f<T>(out[v]);
            out[v] = from_f<T>(o);
        }
    }
}


// ---------------------------------------------------------- space-to-depth --
// Strided RGB-like layers run on the stride x stride super-pixel image
// (DESIGN.md "space-to-depth"): a stride-st RxS conv on C channels equals a
// stride-1 ceil(R/st) x ceil(S/st) conv on st*st*C channels.
// xs[n][i][j][(a*st + b)*C + c] = x[n][st*i + a - pad][st*j + b - pad][c]
// (0 off the image and in the channel padding c' >= st*st*C).  One thread per
// 16-B chunk of xs, so every store is a full vector.
template <class T>
__global__ void s2d_input_kernel(const T* __restrict__ x, T* __restrict__ xs, int chunks, int H, int W, int C,
                                 FastDiv divI, FastDiv divJ, FastDiv divCpp, FastDiv divStc, FastDiv divC, int st,
                                 int pad, int Cs) {
    pdl_entry();
    constexpr int V = 16 / sizeof(T);
    const int stc = (int)divStc.d, real = st * stc;
    // 32-bit index math with multiply-high divisions (the launcher checks the range)
    for (int idx = blockIdx.x * blockDim.x + threadIdx.x; idx < chunks; idx += gridDim.x * blockDim.x) {
        const int pix = (int)divCpp.div((uint32_t)idx);
        const int c0 = (idx - pix * (int)divCpp.d) * V;
        __align__(16) T vals[V];
        if (c0 >= real) {
#pragma unroll
            for (int u = 0; u < V; ++u) vals[u] = from_f<T>(0.f);
        } else {
            const int t = (int)divJ.div((uint32_t)pix), j = pix - t * (int)divJ.d;
            const int n = (int)divI.div((uint32_t)t), i = t - n * (int)divI.d;
            const int h0 = st * i - pad, w0 = st * j - pad;
            int a = (int)divStc.div((uint32_t)c0);
            const int r0 = c0 - a * stc;
            int b = (int)divC.div((uint32_t)r0), c = r0 - b * C;
            const T* xn = x + (size_t)n * H * W * C;
#pragma unroll
            for (int u = 0; u < V; ++u) {
                const int h = h0 + a, w = w0 + b;
                vals[u] = (c0 + u < real && (unsigned)h < (unsigned)H && (unsigned)w < (unsigned)W)
                              ? xn[(h * W + w) * C + c]
                              : from_f<T>(0.f);
                if (++c == C) { c = 0; if (++b == st) { b = 0; ++a; } }
            }
        }
        *reinterpret_cast<uint4*>(xs + (size_t)idx * V) = *reinterpret_cast<const uint4*>(vals);
    }
}

// Space-to-depth filter.  FWD (K-major B of the stride-1 conv on xs, output
// super-pixels of u x u outputs; input super-pixels of f = st*u pixels):
//   out[(uu*u + vv)*K + k][(d*Ds + e)*Cs + (a*f + b)*C + c] = w[k][f*d + a - st*uu][f*e + b - st*vv][c]
// DGRAD (dx super-pixels of f = st*u; K-major B of the transposed conv, N = f*f*C columns of dx):
//   out[(a*f + b)*C + c][(d*Ds + e)*K + k] = w[k][st*d + a - st*(u-1)][st*e + b - st*(u-1)][c]
// Zero where the filter tap falls outside R x S, or in the channel padding.
template <class T>
__global__ void s2d_filter_kernel(const T* __restrict__ w, T* __restrict__ out, int64_t total, int K, int R, int S,
                                  int C, int st, int f, int u, int Dr, int Ds, int Cs, bool dgrad) {
    pdl_entry();
    const int fc = f * C, real = f * fc;
    for (int64_t idx = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; idx < total;
         idx += (int64_t)gridDim.x * blockDim.x) {
        int k, tap, ch, uu = 0, vv = 0;
        if (!dgrad) {
            const int row = Dr * Ds * Cs;
            const int orow = (int)(idx / row);
            const int rem = (int)(idx - (int64_t)orow * row);
            tap = rem / Cs; ch = rem - tap * Cs;
            const int uv = orow / K;
            k = orow - uv * K; uu = uv / u; vv = uv - uu * u;
        } else {
            const int row = Dr * Ds * K;
            ch = (int)(idx / row);
            const int rem = (int)(idx - (int64_t)ch * row);
            tap = rem / K; k = rem - tap * K;
        }
        T v = from_f<T>(0.f);
        if (ch < real) {
            const int d = tap / Ds, e = tap - d * Ds;
            const int a = ch / fc, b = (ch - a * fc) / C, c = ch - a * fc - b * C;
            const int r = dgrad ? st * d + a - st * (u - 1) : f * d + a - st * uu;
            const int s = dgrad ? st * e + b - st * (u - 1) : f * e + b - st * vv;
            if (r >= 0 && r < R && s >= 0 && s < S) v = w[(((int64_t)k * R + r) * S + s) * C + c];
        }
        out[idx] = v;
    }
}

}  // namespace

int launch_im2col(const Geom& g, int32_t b, const void* x, void* col, int32_t kpitch, cudaStream_t st) {
    return g.math == MUCU_MATH_BF16 ? im2col_t<__nv_bfloat16>(g, b, x, col, kpitch, st)
                                    : im2col_t<float>(g, b, x, col, kpitch, st);
}

int launch_pad_filter(const Geom& g, const void* w, void* wpad, int32_t kpitch, cudaStream_t st) {
    const int RSC = g.r * g.s * g.c;
    int grid = grid_for((int64_t)g.k * kpitch, 256);
    if (g.math == MUCU_MATH_BF16)
        launch_pdl(pad_filter_kernel<__nv_bfloat16>, dim3(grid), dim3(256), (size_t)(0), st, (const __nv_bfloat16*)w, (__nv_bfloat16*)wpad, g.k, RSC, kpitch);
    else
        launch_pdl(pad_filter_kernel<float>, dim3(grid), dim3(256), (size_t)(0), st, (const float*)w, (float*)wpad, g.k, RSC, kpitch);
    count_launch();
    return (int)cudaGetLastError();
}

int launch_col2im(const Geom& g, int32_t b, float alpha, const float* dcol, int32_t kpitch, float beta,
                  void* dx, cudaStream_t st) {
    const int64_t pixels = (int64_t)b * g.h * g.w;
    if (g.c < 4) {
        // tiny C (RGB input layer): one thread per dx pixel, all channels in
        // registers; neighbouring threads read neighbouring taps of a dcol row.
        const int grid = grid_for(pixels, 256);
        if (g.math == MUCU_MATH_BF16)
            launch_pdl(col2im_pixel_kernel<__nv_bfloat16>, dim3(grid), dim3(256), (size_t)(0), st, dcol, (__nv_bfloat16*)dx, pixels, g.h, g.w, g.c, g.p,
                                                                    g.q, g.r, g.s, g.pad, g.stride, kpitch, alpha, beta);
        else
            launch_pdl(col2im_pixel_kernel<float>, dim3(grid), dim3(256), (size_t)(0), st, dcol, (float*)dx, pixels, g.h, g.w, g.c, g.p, g.q, g.r,
                                                            g.s, g.pad, g.stride, kpitch, alpha, beta);
        count_launch();
        return (int)cudaGetLastError();
    }
    const bool v4 = g.c % 4 == 0 && kpitch % 4 == 0;
    const int grid = grid_for(pixels * (v4 ? g.c / 4 : g.c), 256);
#define COL2IM(TT, VV)                                                                                            \
    launch_pdl(col2im_taps_kernel<TT, VV>, dim3(grid), dim3(256), (size_t)(0), st, dcol, (TT*)dx, pixels, g.h, g.w, g.c, g.p, g.q, g.r, g.s,   \
                                                     g.pad, g.stride, kpitch, alpha, beta)
    if (g.math == MUCU_MATH_BF16) {
        if (v4) COL2IM(__nv_bfloat16, 4); else COL2IM(__nv_bfloat16, 1);
    } else {
        if (v4) COL2IM(float, 4); else COL2IM(float, 1);
    }
#undef COL2IM
    count_launch();
    return (int)cudaGetLastError();
}

namespace {
__global__ void scale_kernel(float* __restrict__ p, int64_t n, float beta) {
    pdl_entry();
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        p[i] = beta == 0.f ? 0.f : beta * p[i];
}
// Strided DGRAD: dx pixels whose phase ((h+pad) % st, (w+pad) % st) meets no
// filter tap (r0 >= R or s0 >= S, e.g. 3 of 4 pixels of a 1x1 stride-2 layer)
// receive no gradient: zero them (beta = 0) in one pass of 16-B stores.
__global__ void zero_tapless_kernel(uint4* __restrict__ dx, int rows, FastDiv div_cpp, FastDiv div_st, int H, int W,
                                    int R, int S, int pad, int st) {
    pdl_entry();
    // one block per dx pixel row (n, h); a row whose phase meets no tap is zeroed
    // whole, otherwise only the pixels whose column phase meets no tap (the
    // per-element index math uses a multiply-high division: this pass writes
    // up to 3/4 of dx for 1x1 stride-2 layers and was instruction-bound)
    const int cpp = (int)div_cpp.d, per_row = W * cpp;
    for (int row = blockIdx.x; row < rows; row += gridDim.x) {
        const int h = row % H;
        uint4* d = dx + (int64_t)row * per_row;
        if ((h + pad) % st >= R) {
            for (int i = threadIdx.x; i < per_row; i += blockDim.x) d[i] = make_uint4(0u, 0u, 0u, 0u);
            continue;
        }
        for (int i = threadIdx.x; i < per_row; i += blockDim.x) {
            const int wp = (int)div_cpp.div((uint32_t)i) + pad;
            if (wp - (int)div_st.div((uint32_t)wp) * st >= S) d[i] = make_uint4(0u, 0u, 0u, 0u);
        }
    }
}
}  // namespace

int launch_zero_tapless(const Geom& g, int32_t b, void* dx, cudaStream_t st) {
    const int elt = elt_size(g.math);
    if ((g.c * elt) % 16 != 0) return -1;
    const int cpp = g.c * elt / 16;
    const int rows = b * g.h;
    launch_pdl(zero_tapless_kernel, dim3(std::min(rows, 148 * 16)), dim3(256), (size_t)(0), st, (uint4*)dx, rows, FastDiv(cpp), FastDiv(g.stride), g.h, g.w, g.r, g.s, g.pad,
                                                                  g.stride);
    count_launch();
    return (int)cudaGetLastError();
}

namespace {
// One thread per pixel: reads C (< 16 B) channels, writes one 16-B vector.
template <class T>
__global__ void pad_channels_kernel(const T* __restrict__ x, T* __restrict__ xp, int64_t pixels, int C) {
    pdl_entry();
    constexpr int V = 16 / sizeof(T);
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < pixels; i += (int64_t)gridDim.x * blockDim.x) {
        __align__(16) T v[V];
#pragma unroll
        for (int c = 0; c < V; ++c) v[c] = c < C ? x[i * C + c] : from_f<T>(0.f);
        *reinterpret_cast<uint4*>(xp + i * V) = *reinterpret_cast<const uint4*>(v);
    }
}
}  // namespace

// xp[n][h][w'][c'] = x[n][h][w' - pad][c'] (zero outside 0 <= w' - pad < W or
// c' >= C); one 16-B store per thread.
template <typename T>
__global__ void win_pad_kernel(const T* __restrict__ x, T* __restrict__ xp, int units, int W, FastDiv divWp, int C,
                               int pad) {
    pdl_entry();
    constexpr int V = 16 / sizeof(T);  // elements per unit = V / 4 pixels of 4 channels
    for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < units; i += gridDim.x * blockDim.x) {
        const int e0 = i * V;
        const int pix0 = e0 / 4;                           // padded pixel index (n, h, w')
        const int row = (int)divWp.div((uint32_t)pix0);     // (n, h)
        const int w0 = pix0 - row * (int)divWp.d;
        __align__(16) T v[V];
#pragma unroll
        for (int u = 0; u < V; ++u) {
            const int w = w0 + u / 4 - pad, c = u % 4;
            v[u] = (c < C && w >= 0 && w < W) ? x[((size_t)row * W + w) * C + c] : from_f<T>(0.f);
        }
        *reinterpret_cast<uint4*>(xp + (size_t)e0) = *reinterpret_cast<const uint4*>(v);
    }
}
int launch_win_pad(const Geom& g, int32_t b, int Wp, const void* x, void* xp, cudaStream_t st) {
    const int64_t units = (int64_t)b * g.h * Wp * 4 * elt_size(g.math) / 16;
    if (units * (16 / elt_size(g.math)) >= (1LL << 31)) return (int)cudaErrorInvalidValue;
    const int grid = grid_for(units, 256);
    const FastDiv dWp(Wp);
    if (g.math == MUCU_MATH_BF16)
        launch_pdl(win_pad_kernel<__nv_bfloat16>, dim3(grid), dim3(256), (size_t)0, st, (const __nv_bfloat16*)x,
                   (__nv_bfloat16*)xp, (int)units, g.w, dWp, g.c, g.pad);
    else
        launch_pdl(win_pad_kernel<float>, dim3(grid), dim3(256), (size_t)0, st, (const float*)x, (float*)xp,
                   (int)units, g.w, dWp, g.c, g.pad);
    count_launch();
    return (int)cudaGetLastError();
}
int launch_pad_channels(const Geom& g, int32_t b, const void* x, void* xp, cudaStream_t st) {
    const int64_t pixels = (int64_t)b * g.h * g.w;
    const int grid = grid_for(pixels, 256);
    if (g.math == MUCU_MATH_BF16)
        launch_pdl(pad_channels_kernel<__nv_bfloat16>, dim3(grid), dim3(256), (size_t)(0), st, (const __nv_bfloat16*)x, (__nv_bfloat16*)xp, pixels, g.c);
    else
        launch_pdl(pad_channels_kernel<float>, dim3(grid), dim3(256), (size_t)(0), st, (const float*)x, (float*)xp, pixels, g.c);
    count_launch();
    return (int)cudaGetLastError();
}

int launch_scale(int64_t n, float beta, float* p, cudaStream_t st) {
    launch_pdl(scale_kernel, dim3(grid_for(n, 256)), dim3(256), (size_t)(0), st, p, n, beta);
    count_launch();
    return (int)cudaGetLastError();
}

int launch_wg_filter(const Geom& g, bool dgrad, const void* w, void* U, cudaStream_t st) {
    const int O = dgrad ? g.c : g.k, I = dgrad ? g.k : g.c;
    int grid = grid_for((int64_t)O * I, 256);
    if (g.math == MUCU_MATH_BF16)
        launch_pdl(wg_filter_kernel<__nv_bfloat16>, dim3(grid), dim3(256), (size_t)(0), st, (const __nv_bfloat16*)w, (__nv_bfloat16*)U, O, I, g.c, dgrad);
    else
        launch_pdl(wg_filter_kernel<float>, dim3(grid), dim3(256), (size_t)(0), st, (const float*)w, (float*)U, O, I, g.c, dgrad);
    count_launch();
    return (int)cudaGetLastError();
}

// Tile counts: FWD tiles cover the output P x Q; DGRAD tiles cover H x W.
static inline void wg_dims(const Geom& g, bool dgrad, int* IH, int* IW, int* I, int* OH, int* OW, int* O,
                           int* pad) {
    if (!dgrad) { *IH = g.h; *IW = g.w; *I = g.c; *OH = g.p; *OW = g.q; *O = g.k; *pad = g.pad; }
    else        { *IH = g.p; *IW = g.q; *I = g.k; *OH = g.h; *OW = g.w; *O = g.c; *pad = 2 - g.pad; }
}

int launch_wg_input(const Geom& g, bool dgrad, int32_t b, const void* in, void* V, cudaStream_t st) {
    int IH, IW, I, OH, OW, O, pad;
    wg_dims(g, dgrad, &IH, &IW, &I, &OH, &OW, &O, &pad);
    const int TH = (OH + 1) / 2, TW = (OW + 1) / 2;
    const int64_t tiles = (int64_t)b * TH * TW;
    if (I % 4 == 0 && tiles * I / 4 < (1LL << 31)) {
        const uint32_t total = (uint32_t)(tiles * I / 4);
        const int grid4 = grid_for(total, 256);
        const FastDiv dI4((uint32_t)(I / 4)), dTW((uint32_t)TW), dTH((uint32_t)TH);
        const int64_t plane = tiles * I;
        if (g.math == MUCU_MATH_BF16)
            launch_pdl(wg_input4_kernel<__nv_bfloat16>, dim3(grid4), dim3(256), (size_t)0, st,
                       (const __nv_bfloat16*)in, (__nv_bfloat16*)V, total, IH, IW, I, I, (uint32_t)tiles, dI4, dTW,
                       dTH, pad, plane);
        else
            launch_pdl(wg_input4_kernel<float>, dim3(grid4), dim3(256), (size_t)0, st, (const float*)in, (float*)V,
                       total, IH, IW, I, I, (uint32_t)tiles, dI4, dTW, dTH, pad, plane);
        count_launch();
        return (int)cudaGetLastError();
    }
    int grid = grid_for(tiles * I, 256);
    if (g.math == MUCU_MATH_BF16)
        launch_pdl(wg_input_kernel<__nv_bfloat16>, dim3(grid), dim3(256), (size_t)(0), st, (const __nv_bfloat16*)in, (__nv_bfloat16*)V, tiles, IH, IW, I, TH, TW, pad);
    else
        launch_pdl(wg_input_kernel<float>, dim3(grid), dim3(256), (size_t)(0), st, (const float*)in, (float*)V, tiles, IH, IW, I, TH, TW, pad);
    count_launch();
    return (int)cudaGetLastError();
}

int launch_wg_output(const Geom& g, bool dgrad, int32_t b, float alpha, const float* M, float beta, void* out,
                     cudaStream_t st) {
    int IH, IW, I, OH, OW, O, pad;
    wg_dims(g, dgrad, &IH, &IW, &I, &OH, &OW, &O, &pad);
    const int TH = (OH + 1) / 2, TW = (OW + 1) / 2;
    const int64_t tiles = (int64_t)b * TH * TW;
    if (O % 4 == 0 && tiles * O / 4 < (1LL << 31)) {
        const uint32_t total = (uint32_t)(tiles * O / 4);
        const int grid4 = grid_for(total, 256);
        const FastDiv dO4((uint32_t)(O / 4)), dTW((uint32_t)TW), dTH((uint32_t)TH);
        const int64_t plane = tiles * O;
        if (g.math == MUCU_MATH_BF16)
            launch_pdl(wg_output4_kernel<__nv_bfloat16>, dim3(grid4), dim3(256), (size_t)0, st, M,
                       (__nv_bfloat16*)out, total, OH, OW, O, dO4, dTW, dTH, alpha, beta, plane);
        else
            launch_pdl(wg_output4_kernel<float>, dim3(grid4), dim3(256), (size_t)0, st, M, (float*)out, total, OH,
                       OW, O, dO4, dTW, dTH, alpha, beta, plane);
        count_launch();
        return (int)cudaGetLastError();
    }
    int grid = grid_for(tiles * O, 256);
    if (g.math == MUCU_MATH_BF16)
        launch_pdl(wg_output_kernel<__nv_bfloat16>, dim3(grid), dim3(256), (size_t)(0), st, M, (__nv_bfloat16*)out, tiles, OH, OW, O, TH, TW, alpha, beta);
    else
        launch_pdl(wg_output_kernel<float>, dim3(grid), dim3(256), (size_t)(0), st, M, (float*)out, tiles, OH, OW, O, TH, TW, alpha, beta);
    count_launch();
    return (int)cudaGetLastError();
}

int launch_s2d_input(const Geom& g, int32_t b, int f, int I, int J, int Cs, const void* x, void* xs, cudaStream_t st) {
    const int V = 16 / elt_size(g.math);
    const int64_t chunks = (int64_t)b * I * J * (Cs / V);
    if (chunks >= (1LL << 31) || (int64_t)g.h * g.w * g.c >= (1LL << 31)) return (int)cudaErrorInvalidValue;
    const int grid = grid_for(chunks, 256);
    const FastDiv dI(I), dJ(J), dCpp(Cs / V), dStc(f * g.c), dC(g.c);
    if (g.math == MUCU_MATH_BF16)
        launch_pdl(s2d_input_kernel<__nv_bfloat16>, dim3(grid), dim3(256), (size_t)0, st, (const __nv_bfloat16*)x,
                   (__nv_bfloat16*)xs, (int)chunks, g.h, g.w, g.c, dI, dJ, dCpp, dStc, dC, f, g.pad, Cs);
    else
        launch_pdl(s2d_input_kernel<float>, dim3(grid), dim3(256), (size_t)0, st, (const float*)x, (float*)xs,
                   (int)chunks, g.h, g.w, g.c, dI, dJ, dCpp, dStc, dC, f, g.pad, Cs);
    count_launch();
    return (int)cudaGetLastError();
}

int launch_s2d_filter(const Geom& g, bool dgrad, const S2d& z, const void* w, void* out, cudaStream_t st) {
    const int64_t total = dgrad ? (int64_t)z.f * z.f * g.c * z.Dr * z.Ds * g.k
                                : (int64_t)z.u * z.u * g.k * z.Dr * z.Ds * z.Cs;
    const int grid = grid_for(total, 256);
    if (g.math == MUCU_MATH_BF16)
        launch_pdl(s2d_filter_kernel<__nv_bfloat16>, dim3(grid), dim3(256), (size_t)(0), st, (const __nv_bfloat16*)w, (__nv_bfloat16*)out, total,
                                                               g.k, g.r, g.s, g.c, g.stride, z.f, z.u, z.Dr, z.Ds,
                                                               z.Cs, dgrad);
    else
        launch_pdl(s2d_filter_kernel<float>, dim3(grid), dim3(256), (size_t)(0), st, (const float*)w, (float*)out, total, g.k, g.r, g.s, g.c,
                                                       g.stride, z.f, z.u, z.Dr, z.Ds, z.Cs, dgrad);
    count_launch();
    return (int)cudaGetLastError();
}

int launch_wgw_transforms(const Geom& g, int32_t b, const void* x, const void* dy, void* V, void* D, int64_t Tp,
                          cudaStream_t st) {
    const int TH = (g.p + 1) / 2, TW = (g.q + 1) / 2;
    const int64_t tiles = (int64_t)b * TH * TW;
    const int at = 128 / elt_size(g.math);
    const int Cp = (int)align_up((uint64_t)g.c, (uint64_t)at), Kp = (int)align_up((uint64_t)g.k, (uint64_t)at);
    const bool vec = g.c % 4 == 0 && Tp * Cp / 4 < (1LL << 31);
    if (vec) {
        // x transform: 4 channels per thread (vector loads / stores)
        const uint32_t total = (uint32_t)(Tp * Cp / 4);
        const FastDiv dI4((uint32_t)(Cp / 4)), dTW((uint32_t)TW), dTH((uint32_t)TH);
        if (g.math == MUCU_MATH_BF16)
            launch_pdl(wg_input4_kernel<__nv_bfloat16>, dim3(grid_for(total, 256)), dim3(256), (size_t)0, st,
                       (const __nv_bfloat16*)x, (__nv_bfloat16*)V, total, g.h, g.w, g.c, Cp, (uint32_t)tiles, dI4,
                       dTW, dTH, g.pad, Tp * Cp);
        else
            launch_pdl(wg_input4_kernel<float>, dim3(grid_for(total, 256)), dim3(256), (size_t)0, st, (const float*)x,
                       (float*)V, total, g.h, g.w, g.c, Cp, (uint32_t)tiles, dI4, dTW, dTH, g.pad, Tp * Cp);
        count_launch();
    }
    if (g.math == MUCU_MATH_BF16) {
        if (!vec) {
            launch_pdl(wgw_x_kernel<__nv_bfloat16>, dim3(grid_for(Tp * Cp, 256)), dim3(256), (size_t)(0), st,
                (const __nv_bfloat16*)x, (__nv_bfloat16*)V, tiles, Tp, g.h, g.w, g.c, Cp, TH, TW, g.pad);
            count_launch();
        }
        launch_pdl(wgw_dy_kernel<__nv_bfloat16>, dim3(grid_for(Tp * Kp, 256)), dim3(256), (size_t)(0), st, 
            (const __nv_bfloat16*)dy, (__nv_bfloat16*)D, tiles, Tp, g.p, g.q, g.k, Kp, TH, TW);
    } else {
        if (!vec) {
            launch_pdl(wgw_x_kernel<float>, dim3(grid_for(Tp * Cp, 256)), dim3(256), (size_t)(0), st, (const float*)x,
                       (float*)V, tiles, Tp, g.h, g.w, g.c, Cp, TH, TW, g.pad);
            count_launch();
        }
        launch_pdl(wgw_dy_kernel<float>, dim3(grid_for(Tp * Kp, 256)), dim3(256), (size_t)(0), st, (const float*)dy, (float*)D, tiles, Tp, g.p,
                                                                     g.q, g.k, Kp, TH, TW);
    }
    count_launch();
    return (int)cudaGetLastError();
}

// out = alpha * sum_s part[s] + beta * out, splits summed in order (reads of part
// coalesced along n).
__global__ void partial_reduce_kernel(int S, int64_t slot, int ldp, int M, int N, bool transpose,
                                      const float* __restrict__ part, float alpha, float beta, float* __restrict__ out,
                                      const RedTarget red) {
    pdl_entry();
    const int64_t total = (int64_t)M * N;
    for (int64_t idx = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; idx < total;
         idx += (int64_t)gridDim.x * blockDim.x) {
        const int m = (int)(idx / N), n = (int)(idx - (int64_t)m * N);
        const float* p = part + (size_t)m * ldp + n;
        float acc = 0.f;
        // slots summed in order; eight loads in flight per group (the adds stay sequential)
        int s = 0;
        for (; s + 8 <= S; s += 8) {
            float v[8];
#pragma unroll
            for (int u = 0; u < 8; ++u) v[u] = __ldg(p + (size_t)(s + u) * slot);
#pragma unroll
            for (int u = 0; u < 8; ++u) acc += v[u];
        }
        for (; s < S; ++s) acc += __ldg(p + (size_t)s * slot);
        float* d = transpose ? out + (size_t)n * M + m : out + idx;
        const float o = beta != 0.f ? alpha * acc + beta * *d : alpha * acc;
        *d = o;
        if (red.n) red_add(red, d - out, o);  // NEXT-3: the cross-rank dW sum
    }
}

int launch_partial_reduce(int S, int64_t slot, int ldp, int M, int N, bool transpose, const float* part,
                          float alpha, float beta, float* out, cudaStream_t st, const RedTarget* red) {
    RedTarget r = {};
    if (red) r = *red;
    launch_pdl(partial_reduce_kernel, dim3(grid_for((int64_t)M * N, 256)), dim3(256), (size_t)0, st, S, slot, ldp,
               M, N, transpose, part, alpha, beta, out, r);
    count_launch();
    return (int)cudaGetLastError();
}

// Window BackwardFilter partial slots: part[s][m][k] over window rows
// m = (r, atom ja, tap t, channel c) (per_atom = t * cp + c per atom, na atoms per filter
// row) -> dw[k][r][ja*tpa + t][c]; slots summed in order (eight loads in flight),
// padding rows skipped.
__global__ void partial_reduce_win_kernel(int S, int64_t slot, int M, int K, int per_atom, int cp, int na, int R,
                                          int Sf, int C, const float* __restrict__ part, float alpha, float beta,
                                          float* __restrict__ dw, const RedTarget red) {
    pdl_entry();
    const int64_t total = (int64_t)M * K;
    const int64_t RSC = (int64_t)R * Sf * C;
    for (int64_t idx = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; idx < total;
         idx += (int64_t)gridDim.x * blockDim.x) {
        const int m = (int)(idx / K), k = (int)(idx - (int64_t)m * K);
        const int ja = m / per_atom, e = m - ja * per_atom;
        const int t = e / cp, c = e - t * cp;
        const int r = ja / na, sx = (ja - r * na) * (per_atom / cp) + t;
        if (r >= R || sx >= Sf || c >= C) continue;
        const float* p = part + (size_t)m * K + k;
        float acc = 0.f;
        int s = 0;
        for (; s + 8 <= S; s += 8) {
            float v[8];
#pragma unroll
            for (int u = 0; u < 8; ++u) v[u] = __ldg(p + (size_t)(s + u) * slot);
#pragma unroll
            for (int u = 0; u < 8; ++u) acc += v[u];
        }
        for (; s < S; ++s) acc += __ldg(p + (size_t)s * slot);
        float* d = dw + (int64_t)k * RSC + ((int64_t)r * Sf + sx) * C + c;
        const float o = beta != 0.f ? alpha * acc + beta * *d : alpha * acc;
        *d = o;
        if (red.n) red_add(red, d - dw, o);  // NEXT-3: the cross-rank dW sum
    }
}

int launch_partial_reduce_win(int S, int64_t slot, int M, int K, int per_atom, int cp, int na, const Geom& g,
                              const float* part, float alpha, float beta, float* dw, cudaStream_t st,
                              const RedTarget* red) {
    RedTarget r = {};
    if (red) r = *red;
    launch_pdl(partial_reduce_win_kernel, dim3(grid_for((int64_t)M * K, 256)), dim3(256), (size_t)0, st, S, slot, M,
               K, per_atom, cp, na, g.r, g.s, g.c, part, alpha, beta, dw, r);
    count_launch();
    return (int)cudaGetLastError();
}

int launch_wgw_output(const Geom& g, float alpha, const float* M, float beta, float* dw, cudaStream_t st) {
    const int at = 128 / elt_size(g.math);
    const int Cp = (int)align_up((uint64_t)g.c, (uint64_t)at), Kp = (int)align_up((uint64_t)g.k, (uint64_t)at);
    launch_pdl(wgw_out_kernel, dim3(grid_for((int64_t)g.k * g.c, 256)), dim3(256), (size_t)(0), st, M, dw, g.k, g.c, Kp, Cp, alpha, beta);
    count_launch();
    return (int)cudaGetLastError();
}

}  // namespace mucu
