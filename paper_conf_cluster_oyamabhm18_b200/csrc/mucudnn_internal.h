// mucudnn_internal.h -- shared declarations of the library's host runtime and
// kernel launchers (not part of the public ABI; see include/mucudnn.h).
#pragma once
#include <cstdint>
#include <cstddef>

#include "mucudnn.h"

#ifdef __CUDACC__
#include <cstdio>
#include <cuda_runtime.h>
#else
typedef struct CUstream_st* cudaStream_t;
#endif

namespace mucu {

// Records a thread-local error message and returns `s` (printf-style).
mucu_status_t set_error(mucu_status_t s, const char* fmt, ...);

// Process-wide count of kernel launches issued by the library (mucu_launch_count).
void count_launch();

// Layer geometry with derived output extent (reading G1/G3).
struct Geom {
    int32_t n, c, h, w, k, r, s, pad, stride, p, q, math;
};

bool make_geom(const mucu_conv_desc_t* d, Geom* g);
inline int elt_size(int math) { return math == MUCU_MATH_BF16 ? 2 : 4; }
inline uint64_t align_up(uint64_t v, uint64_t a) { return (v + a - 1) / a * a; }
inline int64_t ceil_div(int64_t a, int64_t b) { return (a + b - 1) / b; }

// Algorithm eligibility (UNSUPPORTED reasons) -- shared by workspace sizing,
// the benchmark pass and the executor.
bool algo_eligible(const Geom& g, int type, int algo);
bool is_pointwise(const Geom& g);  // 1x1, stride 1, pad 0: im2col(x) == x
bool small_c_tc(const Geom& g);    // tensor-core math and C*elt < 16 B (RGB input layer)
// Tensor-core I2C BackwardFilter whose im2col is done by the TMA unit into shared memory
// (C a multiple of the 128-B atom, not 1x1): the workspace holds only the per-split
// partial dW slots.
bool i2c_implicit_wgrad(const Geom& g);
// Its partial slots: enough splits to fill every SM with the largest (256 x 256) dW tiles.
int wgrad_implicit_slots(const Geom& g);
// Strided small-C layers whose I2C algorithm runs on the space-to-depth image:
// a stride-1 ceil(R/st) x ceil(S/st) conv over st*st*C channels (padded to
// s2d_channels = a multiple of 128 B).  DGRAD (no padding: the super-pixel
// channels are GEMM columns) needs K to be a multiple of 128 B / elt.
bool s2d_tc(const Geom& g, int type);
// Space-to-depth geometry (FWD / WGRAD; DGRAD uses u = 1 on the dx grid):
// input super-pixels of f = st*u pixels, output super-pixels of u x u outputs
// (u = 2 for stride-2 FWD: N = 4K columns instead of 12 -> 64 padded channels
// per output pixel), Dr x Ds taps, Cs channels, Pu x Qu output super-pixels,
// I x J input super-pixels.
struct S2d { int u, f, Dr, Ds, Cs, Pu, Qu, I, J; };
S2d s2d_geom(const Geom& g, int type);
int s2d_channels(const Geom& g);
inline int s2d_taps(int r, int stride) { return (r + stride - 1) / stride; }
// Window WGRAD (strided small-C layers, I2C algorithm): x copied
// to xp[b][H][Wp][4] (channels zero-padded to 4, `pad` zero columns on the
// left, zeros up to Wp on the right).  GEMM row j = (r, atom, tap, c) of output
// pixel (n,p,q) reads xp[n][st*p + r - pad][st*q + atom*tpa + tap][c]: one
// aw-byte window per (pixel, filter row, atom), windows starting st pixels
// apart -- a plain strided view that TMA tiles directly.
struct Win { int cpx, aw, tpa, na, Wp, M; };  // aw: bytes per swizzle atom (128 / 64 / 32)
bool win_tc(const Geom& g, int type);
Win win_geom(const Geom& g);

// Staged-row BackwardFilter of small-C strided layers: GEMM rows =
// the exact R*S*C taps padded to TR (128-row halves, mt = TR/128), columns = the K
// filters, k-blocks of kd pixels of one output row; x rows staged in chunks of cs
// elements (bch chunks per stage), Ss operand stages, SX x stages.
struct StagedWg { int TR, mt, kd, cs, bch, sx_tx, sx_bytes, tab_bytes, b_bytes, Ss, SX; };
bool staged_wg_geom(const Geom& g, StagedWg* z);
// I2C BackwardFilter of those layers: the staged kernel writes the partial dW tile
// of each of its (up to kPartialSlots) pixel splits to the workspace and a
// reduction kernel sums them in split order (deterministic, all SMs busy).
constexpr int kPartialSlots = 148;

// FFT / FFT_TILING (kernels_fft.cu): F x F real DFT tiles of Th x Tw
// outputs (output = y / dy grid for FWD / WGRAD, dx grid for DGRAD), tiles_y x tiles_x
// tiles per image, bins = F * (F/2 + 1) Hermitian-half frequencies.  false = ineligible
// (MUCU_MATH_F32 and unit stride only; FFT: F <= 32, FFT_TILING: R, S <= 16).
struct FftGeom { int F, Th, Tw, tiles_y, tiles_x; int64_t bins; };
bool fft_geom(const Geom& g, int type, int algo, FftGeom* z);

// Workspace layout of one micro-configuration (all offsets 256-B aligned).
// `fixed` = b-independent prefix (padded filter / Winograd U) computed once per
// call and shared by the call's micro-batches of the same algorithm.
struct WsLayout {
    uint64_t fixed_off, fixed_bytes;  // padded filter (I2C) or U (WG)
    uint64_t a_off, a_bytes;          // col (I2C FWD/WGRAD), dcol (I2C DGRAD), V (WG)
    uint64_t b_off, b_bytes;          // M (WG)
    uint64_t total;
    int32_t kpitch;                   // row pitch (elements) of col / padded filter / dcol
    bool filter_padded;               // I2C: the filter row R*S*C is not 16-B aligned
};
mucu_status_t ws_layout(const Geom& g, int type, int algo, int32_t b, WsLayout* out);

// NEXT-3 reduction target of BackwardFilter (the public mucu_reduce_target_t):
// element-aligned with dw; n = 0: off.
constexpr int kMaxRedRanks = MUCU_MAX_REDUCE_RANKS;
struct RedTarget {
    float* dst[kMaxRedRanks];
    int n;
    int mc;
};

// Per-call executor state (which b-independent workspace prefix is valid).
struct CallCtx {
    int fixed_kind = 0;  // 0 none, 1 padded filter, 2 Winograd U, 3/4 space-to-depth filter, 5 FFT filter spectrum,
                         // 6 FFT BackwardFilter spectrum accumulating over consecutive micro-configs
    const void* fixed_src = nullptr;
    int last_algo = -1;  // algorithm of the previous micro-config (prefix invalidation)
    int next_algo = -1;  // algorithm of the next micro-config of the call (-1: this is the last)
    float fft_beta = 0.f;  // FFT BackwardFilter: beta of the first micro-config of a run (kind 6)
    bool dry = false;    // tensor-core dispatch decisions only, no launch (pre-validation)
    bool deterministic = true;  // BackwardFilter split-K: ordered reduction (default) or L2 atomics
    // NEXT-3: the cross-rank dW sum target (red.n = 0: off), used by the
    // call's last micro-configuration (mc_last); the final dw writer sets mc_fused when
    // it took the reduction in its epilogue.
    RedTarget red = {};
    bool mc_last = false;
    bool mc_fused = false;
};

struct Handle;
// Run one micro-configuration on micro-batch b (pointers already offset).
mucu_status_t run_micro(Handle* h, const Geom& g, int type, int algo, int32_t b, float alpha,
                        const void* in0, const void* in1, float beta, void* out, void* ws,
                        uint64_t ws_bytes, cudaStream_t st, CallCtx* ctx);

#ifdef __CUDACC__
// Division by a run-time constant with a host-computed magic number
// (multiply-high + shift; exact for every 32-bit numerator).
struct FastDiv {
    uint32_t d, m, l;
    FastDiv() = default;
    explicit FastDiv(uint32_t dv) : d(dv), l(0) {
        while ((1ull << l) < dv) ++l;
        m = (uint32_t)((((1ull << 32) * ((1ull << l) - dv)) / dv) + 1);
    }
    __device__ __forceinline__ uint32_t div(uint32_t n) const {
        return (uint32_t)(((uint64_t)__umulhi(n, m) + n) >> l);
    }
};
// NEXT-3: add v at element offset `off` of the reduction target -- one multimem.red
// to a multicast (NVLS) address (NVSwitch adds it into every rank's copy), or one
// red.global.add per rank buffer (peer pointers over NVLink P2P; the rank's own
// buffer at one rank).  Relaxed, system scope: made visible to the peers by the
// release of the barrier (nvls.cu).
__device__ __forceinline__ void red_add(const RedTarget& t, long long off, float v) {
    if (t.mc) {
        asm volatile("multimem.red.relaxed.sys.global.add.f32 [%0], %1;" ::"l"(t.dst[0] + off), "f"(v) : "memory");
    } else {
        for (int r = 0; r < t.n; ++r)
            asm volatile("red.relaxed.sys.global.add.f32 [%0], %1;" ::"l"(t.dst[r] + off), "f"(v) : "memory");
    }
}
__device__ __forceinline__ void red_add4(const RedTarget& t, long long off, float4 v) {  // 16-B aligned
    if (t.mc) {
        asm volatile("multimem.red.relaxed.sys.global.add.v4.f32 [%0], {%1, %2, %3, %4};" ::"l"(t.dst[0] + off),
                     "f"(v.x), "f"(v.y), "f"(v.z), "f"(v.w)
                     : "memory");
    } else {
        for (int r = 0; r < t.n; ++r)
            asm volatile("red.relaxed.sys.global.add.v4.f32 [%0], {%1, %2, %3, %4};" ::"l"(t.dst[r] + off), "f"(v.x),
                         "f"(v.y), "f"(v.z), "f"(v.w)
                         : "memory");
    }
}
#endif

// ---------------------------------------------------------------- kernels --
// All launchers are asynchronous on `st` and return a CUDA error code (0 = ok).
// Ordered split-K turn counters (turns.cu): a launch-private range of `count`
// counters from a static device pool plus a process-unique epoch.  Split s of
// a tile waits for tag(epoch, s - 1) and publishes tag(epoch, s).
struct TurnRange {
    unsigned long long* ctr;
    unsigned long long epoch;
};
int alloc_turns(int64_t count, TurnRange* out);  // cudaError_t
#ifdef __CUDACC__
__host__ __device__ __forceinline__ unsigned long long turn_tag(unsigned long long epoch, int split) {
    return (epoch << 20) + (unsigned long long)split + 1ull;
}
// Watchdog of every spin-wait in the library's kernels: a wait that has not been
// satisfied after kWatchdogNs reports what it waited for and traps (the launch then
// fails with a CUDA error) instead of hanging the device.
constexpr unsigned long long kWatchdogNs = 10ull * 1000 * 1000 * 1000;
__device__ __forceinline__ unsigned long long global_ns() {
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
}
static __device__ __noinline__ void watchdog_trap(const char* what, unsigned long long addr, unsigned long long want,
                                           unsigned long long have) {
    printf("[mucu watchdog] %s wait > %llu s: block (%d,%d,%d) thread %d addr 0x%llx want 0x%llx have 0x%llx\n", what,
           kWatchdogNs / 1000000000ull, (int)blockIdx.x, (int)blockIdx.y, (int)blockIdx.z, (int)threadIdx.x, addr,
           want, have);
    __trap();
}
// One thread waits for the previous split's tag (acquire at gpu scope); the
// caller then synchronises the threads that read dw.
__device__ __forceinline__ void turn_wait(const unsigned long long* c, unsigned long long tag) {
    unsigned long long v;
    unsigned long long t0 = 0;
    for (unsigned n = 0;; ++n) {
        asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(c) : "memory");
        if (v == tag) break;
        __nanosleep(32);
        if ((n & 1023) == 0) {
            const unsigned long long t = global_ns();
            if (!t0) t0 = t;
            else if (t - t0 > kWatchdogNs) watchdog_trap("turn", (unsigned long long)c, tag, v);
        }
    }
}
// One thread publishes after the dw writes of every thread of the group were
// ordered before it by a barrier (release fence is cumulative).
__device__ __forceinline__ void turn_post(unsigned long long* c, unsigned long long tag) {
    asm volatile("fence.acq_rel.gpu;\n\tst.relaxed.gpu.global.u64 [%0], %1;" ::"l"(c), "l"(tag) : "memory");
}
#endif

// SIMT fp32 GEMM-shaped convolution pieces (kernels_simt.cu).
int simt_fwd_ig(const Geom& g, int32_t b, float alpha, const float* x, const float* w, float beta,
                float* y, cudaStream_t st);
int simt_gemm_nt(int64_t M, int64_t N, int64_t K, float alpha, const float* A, int64_t lda,
                 const float* B, int64_t ldb, float beta, float* C, int64_t ldc, int batch,
                 int64_t sA, int64_t sB, int64_t sC, cudaStream_t st);      // C = A[M,K] B[N,K]^T
int simt_gemm_nn(int64_t M, int64_t N, int64_t K, float alpha, const float* A, int64_t lda,
                 const float* B, int64_t ldb, float beta, float* C, int64_t ldc,
                 cudaStream_t st);                                            // C = A[M,K] B[K,N]
int simt_dgrad_ig(const Geom& g, int32_t b, float alpha, const float* dy, const float* w,
                  float beta, float* dx, cudaStream_t st);
// BackwardData of a C <= 4 layer (any math; fp32 FFMA, bf16 / fp32 storage), zero
// workspace: per-phase sub-filter in shared memory, one thread per dx pixel.
// Returns -1 when the layer does not qualify.
int small_c_dgrad(const Geom& g, int32_t b, float alpha, const void* dy, const void* w, float beta, void* dx,
                  cudaStream_t st);
int simt_wgrad(const Geom& g, int32_t b, float alpha, const float* dy, const float* x_or_col,
               bool col_input, int32_t kpitch, float beta, float* dw, int num_sms, cudaStream_t st);

// Element-wise / data-movement kernels (kernels_elem.cu); T = float or bf16 by math.
int launch_im2col(const Geom& g, int32_t b, const void* x, void* col, int32_t kpitch, cudaStream_t st);
int launch_pad_filter(const Geom& g, const void* w, void* wpad, int32_t kpitch, cudaStream_t st);
int launch_col2im(const Geom& g, int32_t b, float alpha, const float* dcol, int32_t kpitch, float beta,
                  void* dx, cudaStream_t st);
int launch_wg_filter(const Geom& g, bool dgrad, const void* w, void* U, cudaStream_t st);
int launch_scale(int64_t n, float beta, float* p, cudaStream_t st);  // p *= beta (beta == 0: p = 0)
// dx = 0 on the pixels of strided-DGRAD phases that meet no filter tap (C*elt % 16 == 0, else -1)
int launch_zero_tapless(const Geom& g, int32_t b, void* dx, cudaStream_t st);
// x[b,H,W,C] -> xp[b,H,W,16/elt] with channels zero-padded to 16 B per pixel.
int launch_pad_channels(const Geom& g, int32_t b, const void* x, void* xp, cudaStream_t st);
// Space-to-depth image xs[b][I][J][Cs] and filters (kernels_elem.cu).
int launch_s2d_input(const Geom& g, int32_t b, int f, int I, int J, int Cs, const void* x, void* xs, cudaStream_t st);
int launch_win_pad(const Geom& g, int32_t b, int Wp, const void* x, void* xp, cudaStream_t st);
int launch_s2d_filter(const Geom& g, bool dgrad, const S2d& z, const void* w, void* out, cudaStream_t st);
int launch_wg_input(const Geom& g, bool dgrad, int32_t b, const void* in, void* V, cudaStream_t st);
int launch_wg_output(const Geom& g, bool dgrad, int32_t b, float alpha, const float* M, float beta,
                     void* out, cudaStream_t st);
// Winograd F(3x3,2x2) BackwardFilter: V[16][Tp][C] = B^T x B and
// D[16][Tp][K] = A dy A^T per 2x2 output tile (rows >= b*T zeroed), then
// dw = alpha * G^T M G + beta * dw with M[16][K][C] fp32.
int launch_wgw_transforms(const Geom& g, int32_t b, const void* x, const void* dy, void* V, void* D, int64_t Tp,
                          cudaStream_t st);
int launch_wgw_output(const Geom& g, float alpha, const float* M, float beta, float* dw, cudaStream_t st);
// out = alpha * sum_{s < S} part[s] + beta * out over an M x N matrix, the split partials
// part[s][m][n] at slot stride `slot` (elements) and row pitch `ldp`; out[m][n] (row pitch
// N), or out[n][m] (row pitch M) when `transpose`.  Summed in split order s = 0, 1, ...
// (deterministic).
// red (NEXT-3): the final values are also added to the cross-rank dW sum (n = 0: off).
int launch_partial_reduce(int S, int64_t slot, int ldp, int M, int N, bool transpose, const float* part,
                          float alpha, float beta, float* out, cudaStream_t st, const RedTarget* red = nullptr);
// The same for the window BackwardFilter's partial tiles (rows = window rows, DESIGN.md
// 6.5; padding rows skipped), out = dw [K][R][S][C].
int launch_partial_reduce_win(int S, int64_t slot, int M, int K, int per_atom, int cp, int na, const Geom& g,
                              const float* part, float alpha, float beta, float* dw, cudaStream_t st,
                              const RedTarget* red = nullptr);
// NEXT-3 (nvls.cu): target[i] += src[i] (16-B vectors where aligned) for the dw writers
// that do not fuse the reduction; and the barrier over the ranks: release-add 1 to
// every flag word in `flags` (one multicast address, or every rank's flag), then wait
// until this rank's own flag reaches `target` (= ranks x barriers so far).
int launch_reduce_push(const float* src, const RedTarget& t, int64_t n, cudaStream_t st);
int launch_reduce_barrier(const RedTarget& flags, const unsigned* own, unsigned target, cudaStream_t st);
// Tensor-core I2C BackwardFilter of large-C layers: partial dW slots reserved in the
// workspace (deterministic split-K over all SMs): ceil(148 / dW tiles of 128 x 128),
// 1 = no partial slots.
int wgrad_partial_slots(const Geom& g);
// F32: M[z][k][c] = sum_t D[z][t][k] * V[z][t][c], z < 16 (SIMT).
int simt_gemm_tt(int64_t K, int64_t C, int64_t Tp, const float* V, const float* D, float* M, int64_t ldt,
                 cudaStream_t st);

// tcgen05 tensor-core path (kernels_tc.cu) for MUCU_MATH_TF32 / MUCU_MATH_BF16:
// runs one micro-configuration; returns a cudaError_t, or -1 if this
// (type, algo, geometry) has no tensor-core implementation.
int tc_run_micro(const Geom& g, int type, int algo, int32_t b, float alpha, const void* in0, const void* in1,
                 float beta, void* out, char* ws, const WsLayout& L, int num_sms, cudaStream_t st,
                 CallCtx* ctx);

// FFT / FFT_TILING micro-configuration (F32): returns 0, a CUDA error, or -1 (ineligible).
struct CallCtx;
int fft_run(const Geom& g, int type, int algo, int32_t b, float alpha, const float* in0, const float* in1, float beta,
            float* out, char* ws, const WsLayout& L, CallCtx* ctx, cudaStream_t st);

}  // namespace mucu
