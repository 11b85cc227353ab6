// kernels_tc.cu -- tcgen05 tensor-core conv-GEMM for sm_100a (MUCU_MATH_TF32 /
// MUCU_MATH_BF16): the contraction step of all three algorithms, and the host-side
// dispatch (tiling, tensor maps, split-K, launch) of one micro-configuration.
//
//   (a) implicit GEMM (zero workspace): the im2col / transposed-conv operand is
//       loaded by TMA in im2col mode (or gathered with cp.async / built in shared
//       memory from TMA-staged rows for small-C strided layers);
//   (b) im2col + GEMM: dense operands loaded with TMA (space-to-depth for strided
//       RGB layers, 6.3);
//   (c) Winograd: 16 independent GEMMs M_xi = V_xi U_xi^T (batched over the tile
//       index), TMA-loaded.
//
// The kernel (tc_gemm_kernel.cuh) is persistent: CTAs walk 128*mt x BN output tiles
// with fp32 accumulators in TMEM.  Warp roles (288 threads; 320 with a TMA warp):
//   warps 0-3  producers (one thread issues TMA; all gather where TMA cannot),
//   warp  4    TMEM allocator + single-thread tcgen05.mma issuer,
//   warps 5-8  epilogue: tcgen05.ld -> registers -> alpha / beta -> global.
// Shared memory is a ring of {A, B} stages guarded by full / empty mbarriers;
// tcgen05.commit releases a stage when its MMAs retire.
//
// Operand layouts (K = reduction):
//   K-major:  rows x 128 B (64 bf16 / 32 fp32 of K), SWIZZLE_128B atoms of 8 rows
//   MN-major: (MN/64 bf16 | MN/32 fp32) atoms, each KB rows x 128 B, SWIZZLE_128B
//             (tf32: 128B_BASE32B)
//
// Backward-filter splits the pixel reduction.  Deterministic mode
// (default): thread-block clusters of cl CTAs (one split each) sum their partial
// tiles over DSMEM in rank order, and split groups add into dw in group order
// behind per-(tile, slab) turn counters (turns.cu), group 0 applying beta; with
// workspace, I2C writes per-split partial slots and a reduction kernel sums them in
// split order -- dw is bitwise reproducible run to run.
// Non-deterministic mode (mucu_set_deterministic(h, 0)): splits add their partials
// with red.global.add after a beta pre-scale.  NEXT-3: the final dw writer also adds
// its values to a cross-rank reduction target (nvls.cu).
#include <cuda.h>
#include <cuda_bf16.h>
#include <cuda_runtime.h>

#include <climits>
#include <cstdio>
#include <cstring>
#include <mutex>
#include <type_traits>

#include "mucudnn_internal.h"

namespace mucu {

namespace {

// ------------------------------------------------------------ PTX helpers --
__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

__device__ __forceinline__ void mbar_init(uint32_t bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(bar), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint32_t bar) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(bar) : "memory");
}
__device__ __forceinline__ void mbar_arrive_tx(uint32_t bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint32_t bar, uint32_t parity) {
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "WAIT_%=:\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t"
        "@!p bra WAIT_%=;\n\t}" ::"r"(bar),
        "r"(parity)
        : "memory");
}
__device__ __forceinline__ void tma_load_2d(uint32_t dst, const CUtensorMap* tm, uint32_t bar, int c0, int c1) {
    asm volatile(
        "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4}], [%2];" ::"r"(dst),
        "l"((uint64_t)tm), "r"(bar), "r"(c0), "r"(c1)
        : "memory");
}
__device__ __forceinline__ void tma_load_3d(uint32_t dst, const CUtensorMap* tm, uint32_t bar, int c0, int c1, int c2) {
    asm volatile(
        "cp.async.bulk.tensor.3d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4, %5}], [%2];" ::"r"(dst),
        "l"((uint64_t)tm), "r"(bar), "r"(c0), "r"(c1), "r"(c2)
        : "memory");
}
__device__ __forceinline__ void tma_load_4d(uint32_t dst, const CUtensorMap* tm, uint32_t bar, int c0, int c1, int c2,
                                            int c3) {
    asm volatile(
        "cp.async.bulk.tensor.4d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4, %5, %6}], [%2];" ::"r"(dst),
        "l"((uint64_t)tm), "r"(bar), "r"(c0), "r"(c1), "r"(c2), "r"(c3)
        : "memory");
}
__device__ __forceinline__ void tma_load_5d(uint32_t dst, const CUtensorMap* tm, uint32_t bar, int c0, int c1, int c2,
                                            int c3, int c4) {
    asm volatile(
        "cp.async.bulk.tensor.5d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4, %5, %6, %7}], [%2];" ::"r"(dst),
        "l"((uint64_t)tm), "r"(bar), "r"(c0), "r"(c1), "r"(c2), "r"(c3), "r"(c4)
        : "memory");
}
// TMA im2col mode (4-D NHWC tensor {C, W, H, N}): pixelsPerColumn consecutive
// pixels starting at (w, h, n) (walking W, then H, then N inside the map's
// bounding box with the map's traversal stride), channelsPerPixel channels
// from c, each read at (w + off_w, h + off_h); zero outside the tensor.
__device__ __forceinline__ void tma_load_im2col_4d(uint32_t dst, const CUtensorMap* tm, uint32_t bar, int c, int w,
                                                   int h, int n, uint16_t off_w, uint16_t off_h) {
    asm volatile(
        "cp.async.bulk.tensor.4d.shared::cluster.global.im2col.mbarrier::complete_tx::bytes"
        " [%0], [%1, {%3, %4, %5, %6}], [%2], {%7, %8};" ::"r"(dst),
        "l"((uint64_t)tm), "r"(bar), "r"(c), "r"(w), "r"(h), "r"(n), "h"(off_w), "h"(off_h)
        : "memory");
}
__device__ __forceinline__ void cp_async16(uint32_t dst, const void* src, bool valid) {
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;" ::"r"(dst), "l"(src), "r"(valid ? 16 : 0) : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void cp_async_wait() { asm volatile("cp.async.wait_group %0;" ::"n"(N) : "memory"); }
__device__ __forceinline__ void fence_proxy_async() { asm volatile("fence.proxy.async.shared::cta;" ::: "memory"); }
__device__ __forceinline__ void tc_fence_before() { asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void tc_fence_after() { asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory"); }

// Shared-memory matrix descriptor (sm_100 version 1).  layout: 2 = SWIZZLE_128B
// (16-B chunks XOR row%8), 1 = SWIZZLE_128B_BASE32B (32-B chunks XOR row%4; the
// only MN-major layout for 32-bit tf32 operands).
__device__ __forceinline__ uint64_t sdesc(uint32_t saddr, uint32_t lbo, uint32_t sbo, uint32_t layout = 2) {
    return (uint64_t)((saddr & 0x3FFFFu) >> 4) | ((uint64_t)((lbo >> 4) & 0x3FFFu) << 16) |
           ((uint64_t)((sbo >> 4) & 0x3FFFu) << 32) | (1ull << 46) | ((uint64_t)layout << 61);
}

template <int ELT>
__device__ __forceinline__ void mma(uint32_t tmem, uint64_t ad, uint64_t bd, uint32_t idesc, uint32_t acc) {
    if constexpr (ELT == 2) {
        asm volatile(
            "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
            "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(tmem),
            "l"(ad), "l"(bd), "r"(idesc), "r"(acc));
    } else {
        asm volatile(
            "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
            "tcgen05.mma.cta_group::1.kind::tf32 [%0], %1, %2, %3, p;\n\t}" ::"r"(tmem),
            "l"(ad), "l"(bd), "r"(idesc), "r"(acc));
    }
}
// Warp-converged variants: all 32 lanes run the issue loop (so descriptors and
// addresses stay warp-uniform and live in uniform registers) and elect.sync
// picks the lane that issues -- the lane-0-only form compiled every MMA into an
// R2UR waterfall loop (~12 instructions of dependent latency per MMA).
template <int ELT>
__device__ __forceinline__ void mma_elect(uint32_t tmem, uint64_t ad, uint64_t bd, uint32_t idesc, uint32_t acc) {
    if constexpr (ELT == 2) {
        asm volatile(
            "{\n\t.reg .pred p, e;\n\tsetp.ne.b32 p, %4, 0;\n\telect.sync _|e, 0xffffffff;\n\t"
            "@e tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(tmem),
            "l"(ad), "l"(bd), "r"(idesc), "r"(acc));
    } else {
        asm volatile(
            "{\n\t.reg .pred p, e;\n\tsetp.ne.b32 p, %4, 0;\n\telect.sync _|e, 0xffffffff;\n\t"
            "@e tcgen05.mma.cta_group::1.kind::tf32 [%0], %1, %2, %3, p;\n\t}" ::"r"(tmem),
            "l"(ad), "l"(bd), "r"(idesc), "r"(acc));
    }
}
__device__ __forceinline__ void mma_commit_elect(uint32_t bar) {
    asm volatile(
        "{\n\t.reg .pred e;\n\telect.sync _|e, 0xffffffff;\n\t"
        "@e tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];\n\t}" ::"r"(bar)
        : "memory");
}
__device__ __forceinline__ void mma_commit(uint32_t bar) {
    asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(bar) : "memory");
}

// 256-bit global stores (sm_100 STG.256): alpha * 16 fp32 accumulators as bf16
// (RNE) / alpha * 8 as fp32; the address must be 32-B aligned.
__device__ __forceinline__ void st256_bf16(__nv_bfloat16* d, const uint32_t* v, float alpha) {
    uint32_t w[8];
#pragma unroll
    for (int u = 0; u < 8; ++u) {
        const __nv_bfloat162 h = __floats2bfloat162_rn(alpha * __uint_as_float(v[2 * u]), alpha * __uint_as_float(v[2 * u + 1]));
        w[u] = *reinterpret_cast<const uint32_t*>(&h);
    }
    asm volatile("st.global.v8.b32 [%0], {%1, %2, %3, %4, %5, %6, %7, %8};" ::"l"(d), "r"(w[0]), "r"(w[1]), "r"(w[2]),
                 "r"(w[3]), "r"(w[4]), "r"(w[5]), "r"(w[6]), "r"(w[7])
                 : "memory");
}
__device__ __forceinline__ void st256_f32(float* d, const uint32_t* v, float alpha) {
    asm volatile("st.global.v8.f32 [%0], {%1, %2, %3, %4, %5, %6, %7, %8};" ::"l"(d), "f"(alpha * __uint_as_float(v[0])),
                 "f"(alpha * __uint_as_float(v[1])), "f"(alpha * __uint_as_float(v[2])), "f"(alpha * __uint_as_float(v[3])),
                 "f"(alpha * __uint_as_float(v[4])), "f"(alpha * __uint_as_float(v[5])), "f"(alpha * __uint_as_float(v[6])),
                 "f"(alpha * __uint_as_float(v[7]))
                 : "memory");
}

#define TMEM_LD32(taddr, v)                                                                                      \
    asm volatile(                                                                                                \
        "tcgen05.ld.sync.aligned.32x32b.x32.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16,%17," \
        "%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];"                                       \
        : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7]),         \
          "=r"(v[8]), "=r"(v[9]), "=r"(v[10]), "=r"(v[11]), "=r"(v[12]), "=r"(v[13]), "=r"(v[14]), "=r"(v[15]),   \
          "=r"(v[16]), "=r"(v[17]), "=r"(v[18]), "=r"(v[19]), "=r"(v[20]), "=r"(v[21]), "=r"(v[22]), "=r"(v[23]), \
          "=r"(v[24]), "=r"(v[25]), "=r"(v[26]), "=r"(v[27]), "=r"(v[28]), "=r"(v[29]), "=r"(v[30]), "=r"(v[31])  \
        : "r"(taddr))

// ----------------------------------------------------------- parameters --
enum AMode : int {
    A_TMA_K2 = 0,      // dense K-major, 2-D map {K, rows}
    A_TMA_K3 = 1,      // dense K-major, batched 3-D map {K, rows, batch}
    A_TMA_MN2 = 2,     // dense MN-major, 2-D map {rows(MN), K}
    A_GATHER_FWD = 3,  // implicit im2col of x, K-major, 16-B vectors (C % KB == 0)
    A_GATHER_DGRAD = 4,// transposed-conv gather of dy, K-major, 16-B vectors (K % KB == 0)
    A_SCALAR_FWD = 5,  // implicit im2col of x, element-wise (any C)
    A_SCALAR_DGRAD = 6,// transposed-conv gather of dy, element-wise (any K)
    A_TMA_IM2COL = 7,  // TMA im2col mode: FWD (x) or stride-1 DGRAD (dy, flipped taps), 128 pixels x KB channels
    A_GATHER_SMALLC = 8, // FWD, C*elt < 16 B (RGB layer): one 16-B chunk per filter tap, channels zero-padded
    A_GATHER_SMALLC_PAD = 9, // same K' layout from a channel-padded copy of x (16 B per pixel): cp.async
    A_HALO = 12,       // stride-1 FWD / DGRAD: per channel chunk, the full source rows a 128*mt-row tile of
                       // the extended output grid touches (one TMA box per row, zero-filled padding); each
                       // tap's A operand is a row-shifted window of that smem halo
    A_TMA_WIN64 = 13,  // A_TMA_WIN with 64-B / 32-B swizzle atoms (BF16; fewer padded taps)
    A_TMA_WIN32 = 14,
    A_TMA_WIN = 11,    // WGRAD window operand, MN-major: rows j = (r, atom, tap, c) of the filter, K = pixels;
                       // one 4-D TMA box per 128-B atom from the overlapping-window view of the padded x
    A_STAGED_FWD = 16, // FWD of small-C strided layers, zero workspace: the x rows of a tile of whole output rows
                       // staged by TMA; builders write the exact-tap (r,s,c) K-major operand
    A_STAGED_WG = 15,  // WGRAD of small-C strided layers, zero workspace: the R x rows a block of KD output
                       // pixels reads are staged by one TMA box; builders write the exact-tap (r,s,c) MN-major
                       // operand from them
};
enum BMode : int {
    B_TMA_K2 = 0,      // dense K-major {K, cols}
    B_TMA_K3 = 1,      // batched K-major {K, cols, batch}
    B_TMA_MN2 = 2,     // dense MN-major {cols(MN), K}
    B_TMA_MN3 = 3,     // DGRAD filter view {C, R*S, K}: B(c, (r,s,k)) = w[k][r][s][c]
    B_GATHER_WG = 4,   // WGRAD implicit im2col of x, MN-major, 16-B vectors (C % atom == 0)
    B_SCALAR_K = 5,    // dense K-major rows with unaligned pitch, element-wise
    B_SCALAR_DGRAD = 6,// DGRAD filter view, element-wise (any C)
    B_SCALAR_WG = 7,   // WGRAD implicit im2col, element-wise (any C)
    B_TMA_IM2COL = 8,  // WGRAD implicit im2col of x by TMA im2col mode, MN-major (KB pixels x 128 B per atom)
    B_RESIDENT = 9,    // whole (padded) filter staged in smem once per CTA (small-C FWD)
    B_GATHER_SMALLC = 10, // WGRAD small C: x pixels as 16-B tap chunks, MN-major
    B_GATHER_SMALLC_PAD = 11, // WGRAD small C from the channel-padded copy of x: cp.async
    B_TMA_DYROW = 12,  // WGRAD dy, MN-major, 3-D map {K, Q, b*P}: k-block = KD pixels of one output row
};
// EPI_D2S: DGRAD on the space-to-depth grid -- row (n, i, j), column
//   (a, b, c) -> dx[n][st*i + a - pad][st*j + b - pad][c] (out-of-image skipped).
// EPI_WGRAD_S2D: column (d, e, (a, b, c')) of the space-to-depth filter ->
//   dw[k][st*d + a][st*e + b][c'] (padding and r >= R / s >= S skipped), reduced.
// EPI_WGRAD_WIN: row j = (r, atom, tap, c) of the window GEMM -> dw[k][r][atom*taps + tap][c], reduced.
// EPI_WGRAD_TAPS: row m = exact tap (r, s, c) -> dw[k][m] (A_STAGED_WG), reduced.
// EPI_WGRAD_PARTIAL: the tile of split z -> out[z][m][n] (fp32, row pitch ldc), plain stores.
enum EpiMode : int { EPI_STORE = 0, EPI_WGRAD_CHAIN = 1, EPI_WGRAD_SMALLC = 2, EPI_D2S = 3, EPI_WGRAD_S2D = 4,
                     EPI_WGRAD_WIN = 5, EPI_WGRAD_TAPS = 6, EPI_WGRAD_PARTIAL = 7 };

struct TcArgs {
    int M, N;                // output rows / cols
    int num_kb;              // k-blocks of the whole reduction
    int num_z;               // batch (WG) or split (WGRAD) count; tiles = mt * nt * num_z
    int kb_per_split;        // WGRAD: k-blocks per blockIdx.z split
    int BN;                  // tile N (multiple of 16, <= 256)
    int stages;
    int tmem_cols;
    int nacc;                // TMEM accumulators (2 = epilogue overlaps the next tile; 1 when mt*BN > 256)
    int km;                  // k-blocks per stage (MN-major BackwardFilter operands; 1 elsewhere)
    int bn_atoms;            // MN-major B atoms per stage = BN * ELT / 128
    int tma_bytes;           // bytes the TMA loads of one stage deliver
    int b_bytes;             // shared-memory bytes of one B stage
    int kred;                // reduction length (elements) for scalar gathers
    // gather geometry (x for FWD/WGRAD, dy for DGRAD)
    const void* gsrc;
    int H, W, C, P, Q, R, S, pad, stride, K;
    // scalar B source
    const void* bsrc;
    int ldb;
    // TMA im2col (A_TMA_IM2COL): DGRAD flips the tap order (r,s) -> (R-1-r, S-1-s)
    // and starts each output pixel at (h + pad - (R-1), w + pad - (S-1)) in dy.
    int im2col_dgrad;
    // Strided DGRAD phase decomposition: dx pixels with (h+pad) % st == r0 and
    // (w+pad) % st == s0 see only taps r = r0 + st*a (a < tapR), s = s0 + st*b
    // (b < tapS), and dy row p = i - a: a stride-1 transposed conv on an
    // (ph_H x ph_W) sub-grid.  tapR/tapS = R/S when not in phase mode.
    int ph_mode, ph_H, ph_W, ph_i0, ph_j0, ph_r0, ph_s0, ph_hb, ph_wb;
    int tapR, tapS;
    // Merged strided-DGRAD launch: ph_n phases (blockIdx-tiles z = phase), each with
    // its own taps / origin / output offset and k-block count; all share ph_H x ph_W
    // and one TMA im2col map (equal start-pixel corners), so one launch covers dx.
    int ph_n, ph_r0v[4], ph_s0v[4], ph_i0v[4], ph_j0v[4], ph_hbv[4], ph_wbv[4], ph_tRv[4], ph_tSv[4], ph_kbv[4];
    int ph_u;                // phase mode: im2col positions advance by ph_u per sub-grid pixel (1 except s2d DGRAD)
    // Small-C layers: K' = (r, s8, c') with taps grouped by 8 per k-block and
    // channels zero-padded to cp = 16 B / elt; s8 = S rounded up to 8.
    int cp, s8;
    int bres_bytes;          // B_RESIDENT: smem bytes of the staged filter
    int max_lag;             // cp.async stages kept in flight per producer thread (<= 6)
    int mt;                  // 128-row halves per tile (1, or 2 for 256-row tiles with narrow N)
    // Space-to-depth layers (EPI_D2S / EPI_WGRAD_S2D): the real stride, C, R, S
    // (the GEMM itself runs on the stride-1 super-pixel geometry).
    int s2_st, s2_C, s2_R, s2_S;
    // EPI_D2S output tensor [*, e_H, e_W, e_C], written at (s2_st*i + a - e_pad, s2_st*j + b - e_pad)
    int e_H, e_W, e_C, e_pad;
    int d2s_rows;            // EPI_D2S by dx rows (beta = 0, one N tile, f*C % 4 == 0)
    // Window WGRAD (A_TMA_WIN / B_TMA_DYROW): 128-B atoms per filter row, q-blocks per output row
    int win_na, win_qb, win_aw;  // + bytes per A swizzle atom (128 / 64 / 32: UMMA layout 2 / 4 / 6)
    int win_box;             // > 0: one 5-D TMA box {atom, KD pixels, na, win_box filter rows} per 128-row half
    int a_box;               // A_TMA_MN2: one 3-D box {atom, KD, atoms} per 128-row half
    int b_box;               // B_TMA_MN3: one 4-D box {atom, 1, KB, bn_atoms} per stage
    int a_merged;            // A_TMA_IM2COL: one im2col box of 128*mt pixels per stage
    // Halo IG (A_HALO): extended grid of hx_H = Ho + R - 1 rows x hx_W (>= Wo + S - 1, multiple of 8)
    // columns per image; source origin offset hx_pe; hx_nch channel chunks of 128 B; halo ring
    int hx_W, hx_H, hx_Ho, hx_Wo, hx_pe, hx_nch, halo_bytes, hstages;
    // Batched split-K (Winograd BackwardFilter): blockIdx-tile batch z = b * zsplit + split;
    // batch b reads operand rows from b * zrows and writes out + b * batch_stride.
    int zsplit, zrows;
    // epilogue
    void* out;
    long long ldc;
    long long batch_stride;  // elements
    float alpha, beta;
    int out_bf16;
    // Cluster split-K BackwardFilter: cl CTAs (one split each) reduce one output tile
    // through DSMEM; split groups of cl are ordered by turn counters (turns.cu), one
    // per (batch, tile, row slab).  stg_bytes: the epilogue's staging over the ring.
    int cl, stg_bytes;
    unsigned long long* tickets;  // ordered split groups: per-tile group tickets (turns.cu pool)
    // A_STAGED_WG: x-row chunks of sx_cs elements (sx_sr = elements per staged row), sx_stages
    // stages of sx_bytes (sx_tx delivered by TMA), kred_taps = R*S*C GEMM rows
    int sx_cs, sx_sr, sx_stages, sx_bytes, sx_tx, kred_taps;
    int atomic;              // non-deterministic split-K: partials added with red.global.add
    int sxw_off;             // A_STAGED_FWD: byte offset of the x-row ring after the resident filter
    int part_rows;           // EPI_WGRAD_PARTIAL: GEMM rows per partial slot (slot = part_rows x ldc floats)
    int m64;                 // MN-major A: the tile's last 128-row half has <= 64 valid rows -> M = 64 MMAs
    unsigned long long* turns;
    unsigned long long epoch;
    // NEXT-3: the cross-rank dW sum, element-aligned with `out`; the final
    // writer of every dw element also adds its value there (multimem.red to a multicast
    // address, or red.global.add per rank buffer; cluster split-K: split group red_group
    // is the final one).  red.n = 0: off.
    RedTarget red;
    int red_group;
};

constexpr int kThreads = 288;  // 4 producer warps, 1 MMA warp, 4 epilogue warps
// A_STAGED_WG adds a TMA warp (9): warps 0-3 and 5-8 build the A operand
constexpr int threads_for(int am) { return (am == 15 || am == 16) ? 320 : kThreads; }

// DGRAD reduction tap index -> filter tap r*S+s (phase mode: the sub-filter
// tap (a,b) is (r0 + st*a, s0 + st*b)).
__device__ __forceinline__ int dgrad_tap_rs(const TcArgs& p, int tap, int r0, int s0, int tapS) {
    if (!p.ph_mode) return tap;
    const int a = tap / tapS, b = tap - a * tapS;
    return (r0 + p.stride * a) * p.S + s0 + p.stride * b;
}

template <int ELT>
struct Elt;
template <>
struct Elt<2> { using T = __nv_bfloat16; static constexpr uint32_t fmt = 1; };
template <>
struct Elt<4> { using T = float; static constexpr uint32_t fmt = 2; };

// Byte offset of element (row, kbyte) inside a K-major SW128 tile.
__device__ __forceinline__ uint32_t kmaj_off(int row, int kbyte) {
    return (uint32_t)((row >> 3) * 1024 + (row & 7) * 128 + ((((kbyte >> 4) ^ (row & 7)) & 7) << 4) + (kbyte & 15));
}
// Byte offset of byte `byte` (0..127) of k-row `krow` inside one MN-major atom
// column: 16-bit types use SWIZZLE_128B (16-B chunk ^ krow%8), 32-bit types
// SWIZZLE_128B_BASE32B (32-B chunk ^ krow%4).
template <int ELT>
__device__ __forceinline__ uint32_t mn_row_off(int krow, int byte) {
    if constexpr (ELT == 2)
        return (uint32_t)(krow * 128 + ((((byte >> 4) ^ (krow & 7)) & 7) << 4) + (byte & 15));
    else
        return (uint32_t)(krow * 128 + ((((byte >> 5) ^ (krow & 3)) & 3) << 5) + (byte & 31));
}
// Byte offset of element (mn, krow) inside an MN-major tile with KB rows per atom.
template <int ELT>
__device__ __forceinline__ uint32_t mnmaj_off(int mn, int krow, int kb_rows) {
    constexpr int per_atom = 128 / ELT;
    const int atom = mn / per_atom;
    return (uint32_t)(atom * kb_rows * 128) + mn_row_off<ELT>(krow, (mn - atom * per_atom) * ELT);
}

template <class T>
__device__ __forceinline__ void st_shared_elt(uint32_t addr, T v);
template <>
__device__ __forceinline__ void st_shared_elt<__nv_bfloat16>(uint32_t addr, __nv_bfloat16 v) {
    unsigned short u = *reinterpret_cast<unsigned short*>(&v);
    asm volatile("st.shared.u16 [%0], %1;" ::"r"(addr), "h"(u) : "memory");
}
template <>
__device__ __forceinline__ void st_shared_elt<float>(uint32_t addr, float v) {
    asm volatile("st.shared.f32 [%0], %1;" ::"r"(addr), "f"(v) : "memory");
}

// ------------------------------------------------------------ the kernel --
#include "tc_gemm_kernel.cuh"

// ------------------------------------------------------------ host side --
typedef CUresult (*EncodeTiledFn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                                  const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                                  CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

EncodeTiledFn get_encode() {
    static EncodeTiledFn fn = nullptr;
    static std::once_flag once;
    std::call_once(once, [] {
        void* p = nullptr;
        cudaDriverEntryPointQueryResult q;
        if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) == cudaSuccess &&
            q == cudaDriverEntryPointSuccess)
            fn = (EncodeTiledFn)p;
    });
    return fn;
}

// Tensor map over a row-major tensor with up to 4 dims (dims[0] contiguous).
bool make_map(CUtensorMap* tm, int elt, const void* base, int rank, const uint64_t* dims, const uint64_t* strides_bytes,
              const uint32_t* box, bool mn_major = false, int swz = 128) {
    // 32-bit MN-major operands need the 32-B-atom swizzle matching SWIZZLE_128B_BASE32B.
    const CUtensorMapSwizzle sw = swz == 0                 ? CU_TENSOR_MAP_SWIZZLE_NONE
                                  : (mn_major && elt == 4) ? CU_TENSOR_MAP_SWIZZLE_128B_ATOM_32B
                                  : swz == 64                ? CU_TENSOR_MAP_SWIZZLE_64B
                                  : swz == 32                ? CU_TENSOR_MAP_SWIZZLE_32B
                                                             : CU_TENSOR_MAP_SWIZZLE_128B;
    EncodeTiledFn enc = get_encode();
    if (!enc) return false;
    cuuint64_t d[5], s[4];
    cuuint32_t b[5], e[5] = {1, 1, 1, 1, 1};
    for (int i = 0; i < rank; ++i) { d[i] = dims[i]; b[i] = box[i]; }
    for (int i = 0; i < rank - 1; ++i) s[i] = strides_bytes[i];
    CUresult r = enc(tm, elt == 2 ? CU_TENSOR_MAP_DATA_TYPE_BFLOAT16 : CU_TENSOR_MAP_DATA_TYPE_FLOAT32, rank,
                     const_cast<void*>(base), d, s, b, e, CU_TENSOR_MAP_INTERLEAVE_NONE, sw,
                     CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    return r == CUDA_SUCCESS;
}

typedef CUresult (*EncodeIm2colFn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                                   const cuuint64_t*, const int*, const int*, cuuint32_t, cuuint32_t,
                                   const cuuint32_t*, CUtensorMapInterleave, CUtensorMapSwizzle,
                                   CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

EncodeIm2colFn get_encode_im2col() {
    static EncodeIm2colFn fn = nullptr;
    static std::once_flag once;
    std::call_once(once, [] {
        void* p = nullptr;
        cudaDriverEntryPointQueryResult q;
        if (cudaGetDriverEntryPoint("cuTensorMapEncodeIm2col", &p, cudaEnableDefault, &q) == cudaSuccess &&
            q == cudaDriverEntryPointSuccess)
            fn = (EncodeIm2colFn)p;
    });
    return fn;
}

// TMA im2col map over an NHWC tensor viewed as {C, W, H, N}.  The bounding box
// of start pixels is [lower, dim - 1 + upper] per spatial dim (W, H order),
// walked with the traversal stride; channelsPerPixel = 128 B of channels.
bool make_im2col_map(CUtensorMap* tm, int elt, const void* base, int C, int W, int H, int N, int lower_w,
                     int lower_h, int upper_w, int upper_h, int pixels, int stride, bool mn_major,
                     bool pixel16 = false) {
    EncodeIm2colFn enc = get_encode_im2col();
    if (!enc) return false;
    if (lower_w < -128 || lower_h < -128 || upper_w > 127 || upper_h > 127 || lower_w > 127 || upper_h < -128)
        return false;
    cuuint64_t d[4] = {(cuuint64_t)C, (cuuint64_t)W, (cuuint64_t)H, (cuuint64_t)N};
    cuuint64_t s[3] = {(cuuint64_t)C * elt, (cuuint64_t)W * C * elt, (cuuint64_t)H * W * C * elt};
    int lo[2] = {lower_w, lower_h}, hi[2] = {upper_w, upper_h};
    cuuint32_t es[4] = {1, (cuuint32_t)stride, (cuuint32_t)stride, 1};
    // pixel16: 16 B of channels per pixel, unswizzled (core-matrix rows of 16 B).
    const CUtensorMapSwizzle sw = pixel16 ? CU_TENSOR_MAP_SWIZZLE_NONE
                                  : (mn_major && elt == 4) ? CU_TENSOR_MAP_SWIZZLE_128B_ATOM_32B
                                                           : CU_TENSOR_MAP_SWIZZLE_128B;
    const cuuint32_t cpp = pixel16 ? (cuuint32_t)(16 / elt) : (cuuint32_t)(128 / elt);
    CUresult r = enc(tm, elt == 2 ? CU_TENSOR_MAP_DATA_TYPE_BFLOAT16 : CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 4,
                     const_cast<void*>(base), d, s, lo, hi, cpp, (cuuint32_t)pixels, es,
                     CU_TENSOR_MAP_INTERLEAVE_NONE, sw, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                     CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    return r == CUDA_SUCCESS;
}

// Dynamic shared memory budget per CTA (227 KB minus alignment slack and barriers).
constexpr int kSmemBudget = 232448 - 1024 - 512;
constexpr int kRingBudget = 200 * 1024;  // operand ring of the default tilings (512-row tiles: +24 KB for a 3rd stage)

int env_int(const char* name, int dflt) {
    const char* e = getenv(name);
    return e ? atoi(e) : dflt;
}

// MUCU_TMA_IM2COL=0 forces the cp.async gather producers (A/B comparison, tests).
bool use_tma_im2col() {
    static int v = -1;
    if (v < 0) {
        const char* e = getenv("MUCU_TMA_IM2COL");
        v = (e && e[0] == '0') ? 0 : 1;
    }
    return v == 1;
}

// Tile N: a multiple of `step` (16 = UMMA granularity at M = 128; an MN-major
// atom when a tile must not split a 128-B channel atom) up to 256, minimising
// the padded columns plus a per-tile overhead (~32 columns, or the A rows a
// tile re-reads); ties -> larger.
// With mtiles > 0 (persistent FWD / DGRAD launches) the cost counts whole
// waves of tiles over the SMs: time ~ waves x (bn + 128), so e.g. ResNet-50
// layer4 (98 row tiles, N = 512) takes 3 x 192 (2 waves) instead of 2 x 256
// (196 tiles = 1.3 waves): DGRAD 0.095 -> 0.077 ms.
int g_num_sms = 148;
int pick_bn(int N, int step = 32, int overhead = 32, int max_bn = 256, int64_t mtiles = 0) {
    step = std::max(step, 32);  // the epilogue drains TMEM in 32-column chunks
    int best = step;
    int64_t best_cost = INT64_MAX;
    const bool waves = mtiles > 0;
    for (int bn = step; bn <= max_bn; bn += step) {
        const int64_t nt = ceil_div(N, bn);
        // per-tile cost in wave mode: narrow tiles run well below the MMA rate of wide
        // ones (one 128 x 64 chain ~ 0.7x the time of a 128 x 256 one), hence +128
        const int64_t cost = waves ? ceil_div(mtiles * nt, g_num_sms) * (bn + 128) : nt * (bn + overhead);
        if (cost <= best_cost) { best = bn; best_cost = cost; }
    }
    return best;
}

// Arguments of the A operand's TMA im2col map (re-encoded with 128*mt pixels per
// box once the tile height is known: one transaction per stage instead of mt).
struct Im2colArgs {
    int valid, elt, C, W, H, N, lw, lh, uw, uh, stride;
    const void* base;
};
struct Launch {
    TcArgs a;
    CUtensorMap ta, tb;
    dim3 grid;
    Im2colArgs ia;
    // NEXT-3: the call's reduction target (last micro-batch only), its local dw and the
    // executor's "fused" flag (set when this launch writes dw and takes the reduction)
    const RedTarget* red;
    const void* mc_local;
    bool* mc_fused;
};

template <int ELT, int AM, int BM_, int EPI>
int launch_t(Launch& L, cudaStream_t st, bool dry) {
    auto kern = tc_conv_gemm<ELT, AM, BM_, EPI>;
    L.a.a_merged = 0;
    if (AM == A_TMA_IM2COL && L.a.mt > 1 && L.ia.valid && env_int("MUCU_A_MERGE", 1)) {
        const Im2colArgs& q = L.ia;
        CUtensorMap tmp;
        if (make_im2col_map(&tmp, q.elt, q.base, q.C, q.W, q.H, q.N, q.lw, q.lh, q.uw, q.uh, 128 * L.a.mt, q.stride,
                            false)) {
            L.ta = tmp;
            L.a.a_merged = 1;
        }
    }
    const int a_stage = AM == A_HALO ? 0 : L.a.mt * 128 * 128;
    const int ring = L.a.hstages * L.a.halo_bytes + L.a.stages * L.a.km * (a_stage + L.a.b_bytes) + L.a.bres_bytes;
    const int smem =
        1024 + std::max(ring, L.a.stg_bytes) + (2 * L.a.stages + 6 + 2 * L.a.hstages + 2 * L.a.sx_stages) * 8 + 64;
    if (smem > 232448) return -1;
    constexpr bool SPLITK = (EPI == EPI_WGRAD_CHAIN || EPI == EPI_WGRAD_SMALLC || EPI == EPI_WGRAD_S2D ||
                             EPI == EPI_WGRAD_WIN || EPI == EPI_WGRAD_TAPS || EPI == EPI_WGRAD_PARTIAL);
    if (!SPLITK && L.a.cl) return -1;
    L.a.turns = nullptr;
    L.a.epoch = 0;
    L.a.red.n = 0;
    L.a.red_group = 0;
    if (dry) return 0;
    // NEXT-3: the launch that writes the call's dw in the last micro-batch is its final
    // writer (one dw-writing launch per micro-configuration; split-K groups ordered):
    // fuse the cross-rank reduction into its epilogue.  Atomic split-K partials and
    // batched (Winograd) outputs are not final values: the executor pushes dw instead.
    if (SPLITK && EPI != EPI_WGRAD_PARTIAL && L.red && L.a.out == L.mc_local && !L.a.atomic && !L.a.zsplit) {
        L.a.red = *L.red;
        L.a.red_group = L.a.cl ? L.a.num_z / L.a.cl - 1 : 0;
        *L.mc_fused = true;
    }
    if (SPLITK && L.a.atomic && L.a.beta != 1.f) {
        // split partials are added with L2 reductions: apply beta to the output first
        int64_t extent;
        if (L.a.zsplit) extent = (int64_t)(L.a.num_z / L.a.zsplit) * L.a.batch_stride;
        else if (EPI == EPI_WGRAD_WIN || EPI == EPI_WGRAD_TAPS) extent = (int64_t)L.a.N * L.a.ldc;
        else extent = (int64_t)L.a.M * L.a.ldc;
        const int e = launch_scale(extent, L.a.beta, (float*)L.a.out, st);
        if (e) return e;
    }
    // Cluster split-K with more split groups than one: a turn counter per (batch,
    // tile, row slab) orders the groups' additions into dw.
    if (SPLITK && L.a.cl) {
        const int64_t splits = L.a.zsplit ? L.a.zsplit : L.a.num_z;
        L.a.tickets = nullptr;
        if (splits > L.a.cl) {
            const int64_t per_z = ceil_div(L.a.M, 128 * L.a.mt) * ceil_div(L.a.N, L.a.BN);
            TurnRange tr, tk;
            int e = alloc_turns(per_z * (L.a.num_z / splits) * L.a.cl, &tr);
            if (!e) e = alloc_turns(per_z * (L.a.num_z / splits), &tk);
            if (e) return e;
            L.a.turns = tr.ctr;
            L.a.epoch = tr.epoch;
            L.a.tickets = tk.ctr;
        }
    }
    static int configured = 0;  // per instantiation
    if (configured < smem) {
        cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, 232448);
        if (e) return (int)e;
        if (SPLITK) cudaFuncSetAttribute(kern, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
        configured = 232448;
    }
    // Programmatic dependent launch (MUCU_PDL=0 disables): the kernel may start
    // (prologue only -- it executes griddepcontrol.wait before touching global
    // memory) while the previous kernel on the stream drains its last wave.
    static const int pdl = env_int("MUCU_PDL", 1);
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = L.grid;
    cfg.blockDim = dim3(threads_for(AM));
    cfg.dynamicSmemBytes = (size_t)smem;
    cfg.stream = st;
    cudaLaunchAttribute attr[2];
    int na = 0;
    if (pdl) {
        attr[na].id = cudaLaunchAttributeProgrammaticStreamSerialization;
        attr[na].val.programmaticStreamSerializationAllowed = 1;
        ++na;
    }
    if (L.a.cl) {
        attr[na].id = cudaLaunchAttributeClusterDimension;
        attr[na].val.clusterDim.x = (unsigned)L.a.cl;
        attr[na].val.clusterDim.y = 1;
        attr[na].val.clusterDim.z = 1;
        ++na;
    }
    cfg.attrs = attr;
    cfg.numAttrs = na;
    cudaError_t le = cudaLaunchKernelEx(&cfg, kern, L.a, L.ta, L.tb);
    if (le) return (int)le;
    count_launch();
    return (int)cudaGetLastError();
}

// CTAs of ~200 KB shared memory that can be resident at once when launched in
// clusters of cl (GPC packing; 0 = cluster size not launchable).  Cached.
__global__ void cluster_probe_kernel() {}
int cluster_capacity(int cl) {
    static int cache[17] = {0};
    if (cl <= 1) return g_num_sms;
    if (cl > 16) return 0;
    if (cache[cl]) return cache[cl] > 0 ? cache[cl] : 0;
    const int sm = 200 * 1024;
    cudaFuncSetAttribute(cluster_probe_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, sm);
    cudaFuncSetAttribute(cluster_probe_kernel, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3((unsigned)(cl * 64));
    cfg.blockDim = dim3(kThreads);
    cfg.dynamicSmemBytes = sm;
    cudaLaunchAttribute at;
    at.id = cudaLaunchAttributeClusterDimension;
    at.val.clusterDim.x = (unsigned)cl;
    at.val.clusterDim.y = 1;
    at.val.clusterDim.z = 1;
    cfg.attrs = &at;
    cfg.numAttrs = 1;
    int n = 0;
    if (cudaOccupancyMaxActiveClusters(&n, cluster_probe_kernel, &cfg) != cudaSuccess || n <= 0) {
        cudaGetLastError();
        n = 0;
    }
    cache[cl] = n > 0 ? n * cl : -1;
    return n * cl;
}

void size_stages(TcArgs& a) {
    a.nacc = a.mt * a.BN <= 256 ? 2 : 1;
    const int cols = a.nacc * a.mt * a.BN;  // accumulator buffers x mt halves
    a.tmem_cols = cols <= 64 ? 64 : cols <= 128 ? 128 : cols <= 256 ? 256 : 512;
    if (a.km < 1) a.km = 1;
    const int stage_bytes = a.km * (a.mt * 128 * 128 + a.b_bytes);
    a.stages = std::min(env_int("MUCU_MAX_STAGES", 8), (kRingBudget + (a.mt == 4 ? 24 * 1024 : 0)) / stage_bytes);
    if (a.stages < 2) a.stages = 2;
}

void finalize_tiling(Launch& L, int elt, int step = 32, int batch = 1) {
    TcArgs& a = L.a;
    a.BN = pick_bn(a.N, step, 32, 256, ceil_div(a.M, 128) * batch);
    if (const int fb = env_int("MUCU_FORCE_BN", 0)) a.BN = std::max(step, fb - fb % step);
    a.bn_atoms = (a.BN * elt + 127) / 128;
    a.b_bytes = std::max(a.BN * 128, a.bn_atoms * (128 / elt) * 128);
    a.mt = 1;
    size_stages(a);
}

// 256- or 512-row tiles (two or four 128-row accumulators sharing each B tile)
// for narrow N: a chain of dependent MMAs into one accumulator runs at one MMA
// per ~250 cycles whatever N is (measured: N = 64 -> 459 TF/s with one chain,
// 570 with two; N = 256 -> 1294), so short-N tiles need several independent
// chains in flight.  TMA-fed K-major A operands only; needs at least one tile
// per SM.
void use_mt2(Launch& L, int num_sms) {
    TcArgs& a = L.a;
    // Wide tiles (128 < BN <= 192): 256 x BN needs one accumulator set (the epilogue
    // no longer overlaps the next tile), worth it for long reductions only; measured
    // AlexNet conv2 FWD / conv3 DGRAD 0.19 / 0.22 -> 0.16 / 0.17 ms, while BN = 256
    // (one 128 x 256 chain is already near the MMA floor) got slower.
    const bool wide_ok = a.num_kb >= 32 && a.BN <= 192;
    if ((a.BN > 128 && !wide_ok) || env_int("MUCU_MT2", 1) == 0) return;
    const int force = env_int("MUCU_FORCE_MT", 0);  // tests: exercise 256/512-row tiles on small shapes
    if (force == 4 && a.BN <= 64) num_sms = 1;
    if (force == 2) { a.mt = 2; size_stages(a); return; }
    if (a.BN <= 64 && ceil_div(a.M, 512) >= num_sms) {
        a.mt = 4;
        size_stages(a);
        return;
    }
    if (ceil_div(a.M, 256) < num_sms) return;
    a.mt = 2;
    size_stages(a);
}

// Halo implicit GEMM geometry for a stride-1 conv viewed as a
// correlation of a source tensor [b][Hs][Ws][Cs] (x for FWD, dy for DGRAD) with
// R x S taps at origin offset pe over an Ho x Wo output grid.  Returns false
// when the halo ring does not fit next to two B stages.
bool halo_setup(TcArgs& a, int elt, int b, int Ho, int Wo, int R, int S, int pe, int Cs) {
    // Opt-in (MUCU_HALO=1): measured slower than the TMA-im2col tiles on every
    // AlexNet / ResNet layer; kept as a tested alternative producer.
    if (env_int("MUCU_HALO", 0) == 0) return false;
    const int KB = 128 / elt;
    if (Cs % KB) return false;
    a.hx_W = (int)align_up((uint64_t)(Wo + S - 1), 8);
    a.hx_H = Ho + R - 1;
    a.hx_Ho = Ho; a.hx_Wo = Wo; a.hx_pe = pe;
    a.hx_nch = Cs / KB;
    if (a.hx_W > 256) return false;  // one TMA box per row
    a.M = (int)std::min<int64_t>((int64_t)b * a.hx_H * a.hx_W, INT32_MAX);
    if ((int64_t)b * a.hx_H * a.hx_W > INT32_MAX) return false;
    const int rows = 128 * a.mt;
    const int nr = (a.hx_W - 8 + rows - 1 + (R - 1) * a.hx_W + S - 1) / a.hx_W + 1;
    a.halo_bytes = (int)align_up((uint64_t)nr * a.hx_W * 128, 1024);
    a.hstages = std::max(1, std::min(4, env_int("MUCU_HSTAGES", 2)));
    a.tapR = R; a.tapS = S;
    a.num_kb = a.hx_nch * R * S;
    const int budget = 200 * 1024 - a.hstages * a.halo_bytes;
    if (budget < 2 * a.b_bytes) return false;
    a.stages = std::min(env_int("MUCU_MAX_STAGES", 8), budget / a.b_bytes);
    return true;
}

}  // namespace

// ====================================================== micro-config run ==
// Returns cudaError_t, or -1 when a shape has no tensor-core path.
int tc_run_micro(const Geom& g, int type, int algo, int32_t b, float alpha, const void* in0, const void* in1,
                 float beta, void* out, char* ws, const WsLayout& WL, int num_sms, cudaStream_t st,
                 CallCtx* ctx) {
    // Dry run (executor pre-validation): every host decision and tensor-map
    // encoding, no launch.
    const bool dry = ctx->dry;
#define DRY(x) (dry ? 0 : (x))
    const int elt = elt_size(g.math);
    const int KB = 128 / elt;
    const int atom = 128 / elt;
    g_num_sms = num_sms;
    const bool bf = g.math == MUCU_MATH_BF16;
    const int64_t PQ = (int64_t)g.p * g.q, HW = (int64_t)g.h * g.w;
    const int RS = g.r * g.s;
    const int64_t RSC = (int64_t)RS * g.c;
    Launch L;
    std::memset(&L, 0, sizeof(L));
    TcArgs& A = L.a;
    A.km = 1;
    A.H = g.h; A.W = g.w; A.C = g.c; A.P = g.p; A.Q = g.q; A.R = g.r; A.S = g.s; A.pad = g.pad;
    A.stride = g.stride; A.K = g.k;
    A.tapR = g.r; A.tapS = g.s; A.ph_u = 1;
    A.max_lag = std::min(6, std::max(1, env_int("MUCU_MAX_LAG", 6)));
    A.alpha = alpha; A.beta = beta; A.out = out; A.out_bf16 = bf ? 1 : 0;
    if (type == MUCU_BWD_FILTER && ctx->red.n && ctx->mc_last) {
        L.red = &ctx->red; L.mc_local = out; L.mc_fused = &ctx->mc_fused;
    }
    // partial-slot reductions are the final writer of dw: they take the cross-rank sum
    const RedTarget* const mc_reduce = L.red;
    auto note_fused = [&]() { if (mc_reduce && !dry) ctx->mc_fused = true; };
    auto map2 = [&](CUtensorMap* tm, const void* base, uint64_t d0, uint64_t d1, uint64_t pitch_elems, uint32_t b0,
                    uint32_t b1, bool mn = false) {
        uint64_t dims[2] = {d0, d1}, str[1] = {pitch_elems * elt};
        uint32_t box[2] = {b0, b1};
        return make_map(tm, elt, base, 2, dims, str, box, mn);
    };
    auto map3 = [&](CUtensorMap* tm, const void* base, uint64_t d0, uint64_t d1, uint64_t d2, uint64_t s1,
                    uint64_t s2, uint32_t b0, uint32_t b1, uint32_t b2, bool mn = false) {
        uint64_t dims[3] = {d0, d1, d2}, str[2] = {s1 * elt, s2 * elt};
        uint32_t box[3] = {b0, b1, b2};
        return make_map(tm, elt, base, 3, dims, str, box, mn);
    };
    // DGRAD filter view {C, R*S, K} as the MN-major B operand: with C and the tile N
    // multiples of the 128-B atom, a 4-D view {atom element, tap, k, atom index} loads
    // the stage's bn_atoms atoms in one TMA box (measured: AlexNet TF32 conv3-5 DGRAD
    // -27..30 %, BF16 -11..14 %, ResNet-50 layer3/4 DGRAD -10..17 %).
    auto map_w_box = [&](const void* w) {
        A.b_box = 0;
        if (g.c % atom || A.BN % atom || !env_int("MUCU_B_BOX", 1)) return;
        uint64_t dims[4] = {(uint64_t)atom, (uint64_t)g.r * g.s, (uint64_t)g.k, (uint64_t)(g.c / atom)};
        uint64_t str[3] = {(uint64_t)g.c * elt, (uint64_t)g.r * g.s * g.c * elt, 128};
        uint32_t box[4] = {(uint32_t)atom, 1, (uint32_t)KB, (uint32_t)A.bn_atoms};
        CUtensorMap tmp;
        if (make_map(&tmp, elt, w, 4, dims, str, box, true)) { L.tb = tmp; A.b_box = 1; }
    };
    // Dense MN-major B operand (rows of `pitch` elements, N = the contiguous dim):
    // a 3-D view {atom element, k row, atom index} loads the stage's bn_atoms atoms in
    // one TMA box when N, the tile N and the pitch are multiples of the 128-B atom.
    auto map_mn_box = [&](const void* base, uint64_t ncols, uint64_t krows, uint64_t pitch, int krows_box) {
        A.b_box = 0;
        if (ncols % atom || pitch % atom || A.BN % atom || !env_int("MUCU_B_BOX", 1)) return;
        uint64_t dims[3] = {(uint64_t)atom, krows, ncols / atom};
        uint64_t str[2] = {pitch * elt, 128};
        uint32_t box[3] = {(uint32_t)atom, (uint32_t)krows_box, (uint32_t)A.bn_atoms};
        CUtensorMap tmp;
        if (make_map(&tmp, elt, base, 3, dims, str, box, true)) { L.tb = tmp; A.b_box = 1; }
    };
    auto im2col_a = [&](int e, const void* base, int C, int W, int H, int N, int lw, int lh, int uw, int uh, int pixels,
                        int stride, bool mn) {
        L.ia = Im2colArgs{1, e, C, W, H, N, lw, lh, uw, uh, stride, base};
        return make_im2col_map(&L.ta, e, base, C, W, H, N, lw, lh, uw, uh, pixels, stride, mn);
    };
    // Persistent launch: one CTA per SM (at most one per tile).
    auto grid2 = [&](int batch) {
        A.num_z = batch;
        const int64_t tiles = ceil_div(A.M, 128 * A.mt) * ceil_div(A.N, A.BN) * batch;
        L.grid = dim3((unsigned)std::max<int64_t>(1, std::min<int64_t>(tiles, num_sms)));
    };
    // BackwardFilter tiling: output rows = K (filter count), columns = the
    // filter taps, reduction = pixels split across CTAs (~2 waves, >= 16
    // k-blocks each).  TMA-fed B operands take 256-row tiles when they cover
    // K without waste, so each B tile is read once per 256 output rows.
    // TMA-only operands (tma = true) also take 256-row tiles and stages of
    // km k-blocks: fewer, larger TMA transactions (the TMA issue rate, not
    // bytes, bounds these MN-major loads), as deep as two stages allow.
    // Split of a BackwardFilter reduction of nkb stages over `tiles` output tiles.
    auto apply_split = [&](int64_t tiles, int64_t nkb, int batches, bool one_unit = false) {
        // Split of the pixel reduction (deterministic): S = cl * G CTAs per
        // tile; clusters of cl reduce their partials through DSMEM (+R) and the G groups
        // add into dw in a fixed order (+L per hand-over).  Cost in stages of km
        // k-blocks: waves of the CTAs that fit at once (GPC packing of clusters) x
        // (stages per split + E for pipeline fill and the epilogue).
        const double E = env_int("MUCU_SPLIT_E", 16) / (double)A.km;
        const double R = env_int("MUCU_CLUSTER_R", 6) / (double)A.km;
        const double Lg = env_int("MUCU_CHAIN_L", 8) / (double)A.km;
        const int force_cl = env_int("MUCU_FORCE_CL", 0), force_g = env_int("MUCU_FORCE_G", 0);  // tests
        int64_t b_s = 1;
        int b_cl = 0;
        double best = force_cl ? 1e30 : (double)ceil_div(tiles, num_sms) * ((double)nkb + E);
        if (!ctx->deterministic) {
            // non-deterministic mode: persistent CTAs, splits reduced with fp32 L2 atomics
            A.atomic = 1;
            int64_t smax = std::min<int64_t>(std::max<int64_t>(1, nkb / 4), 4LL * num_sms);
            if (one_unit) smax = std::min<int64_t>(smax, std::max<int64_t>(1, num_sms / tiles));
            for (int64_t sp = 1; sp <= smax; ++sp) {
                const double cost = (double)ceil_div(tiles * sp, num_sms) * ((double)ceil_div(nkb, sp) + E);
                if (cost < best - 1e-9) { best = cost; b_s = sp; }
            }
            A.num_kb = (int)nkb;
            A.kb_per_split = (int)ceil_div(nkb, b_s);
            b_s = ceil_div(nkb, A.kb_per_split);
            A.cl = 0;
            A.stg_bytes = 0;
            A.zsplit = batches > 1 ? (int)b_s : 0;
            grid2((int)(batches * b_s));
            if (b_s == 1) A.atomic = 0;
            return;
        }
        for (int cl = 2; cl <= 16; cl *= 2) {
            if (force_cl && cl != force_cl) continue;
            const int cap = cluster_capacity(cl);
            if (cap <= 0) continue;
            for (int64_t G = 1;; ++G) {
                const int64_t sp = cl * G;
                if (sp > std::max<int64_t>(2, nkb / 2) || sp > 1024) break;
                if (force_g && G != force_g) continue;
                const double cost = (double)ceil_div(tiles * sp, cap) * ((double)ceil_div(nkb, sp) + E) + R +
                                    (double)(G - 1) * Lg;
                if (cost < best - 1e-9) { best = cost; b_s = sp; b_cl = cl; }
            }
        }
        A.num_kb = (int)nkb;
        A.kb_per_split = (int)ceil_div(nkb, b_s);
        A.cl = b_s > 1 ? b_cl : 0;
        if (env_int("MUCU_LOG_TILING", 0))
            fprintf(stderr, "[mucu] wgrad M=%d N=%d mt=%d BN=%d km=%d tiles=%lld nkb=%lld -> S=%lld cl=%d cap=%d cost=%.1f\n",
                    A.M, A.N, A.mt, A.BN, A.km, (long long)tiles, (long long)nkb, (long long)b_s, A.cl,
                    A.cl ? cluster_capacity(A.cl) : num_sms, best);
        A.zsplit = batches > 1 ? (int)b_s : 0;
        if (A.cl) {
            // one unit per CTA: grid = tiles x splits (a multiple of the cluster size)
            A.num_z = (int)(batches * b_s);
            A.stg_bytes = 128 * A.mt * (A.BN + 4) * 4;
            L.grid = dim3((unsigned)(tiles * b_s));
        } else {
            A.stg_bytes = 0;
            grid2(batches);
        }
    };
    auto wgrad_tiling = [&](int step, bool tma, int qrow = 0, int km_max = 4, int batches = 1) {
        A.mt = (tma && A.M > 128 && (A.M <= 256 || A.M % 256 == 0 || (qrow && A.M % 256 > 128)) &&
                env_int("MUCU_MT2", 1)) ? 2 : 1;
        // 256-row tiles keep BN <= 128 so that two stages of two k-blocks fit
        // (measured: km = 2 beats BN = 256 with km = 1 on every AlexNet/ResNet layer)
        A.BN = pick_bn(A.N, step, 128 * A.mt, A.mt == 2 ? std::max(128, step) : 256);
        if (const int fb = env_int("MUCU_FORCE_BN", 0)) A.BN = std::max(std::max(step, 32), fb - fb % step);
        A.bn_atoms = (A.BN * elt + 127) / 128;
        A.b_bytes = std::max(A.BN * 128, A.bn_atoms * (128 / elt) * 128);
        A.km = 1;
        if (tma) {
            const int base = A.mt * 128 * 128 + A.b_bytes;
            while (A.km < km_max && 2 * (2 * A.km) * base <= 200 * 1024 && KB * 2 * A.km <= 256 &&
                   (qrow == 0 || KB * 2 * A.km <= (int)align_up((uint64_t)qrow, (uint64_t)KB)))
                A.km *= 2;
            // window operand (qrow > 0), BF16: 64-pixel k-blocks already make large boxes;
            // km = 1 keeps 5 ring stages instead of 2 (ResNet conv1 WGRAD -6 %; TF32's
            // 32-pixel blocks need km = 2)
            if (qrow && elt == 2 && env_int("MUCU_WIN_KM1", 1)) A.km = 1;
            if (const int km = env_int("MUCU_KM", 0)) A.km = km;
        }
        size_stages(A);
        // one row tile whose last 128-row half holds <= 64 filters (K = 64, 192, ...): that
        // half issues M = 64 MMAs (the MN-major dy operand is read for 64 rows, not 128)
        A.m64 = !qrow && A.M <= 128 * A.mt && A.M - 128 * (A.mt - 1) <= 64 && env_int("MUCU_M64", 1);
        const int64_t tiles = ceil_div(A.N, A.BN) * ceil_div(A.M, 128 * A.mt) * batches;
        // qrow > 0: k-blocks are KD-pixel pieces of output rows of qrow pixels (window WGRAD)
        if (qrow) A.win_qb = (int)ceil_div(qrow, KB * A.km);
        const int64_t nkb = qrow ? (int64_t)b * g.p * A.win_qb : ceil_div(A.kred, KB * A.km);
        apply_split(tiles, nkb, batches);
    };
    const bool Aok = (g.c % KB) == 0;  // vector gathers over C
    int err = 0;
#define LAUNCH(AMODE, BMODE, EPIM) \
    (elt == 2 ? launch_t<2, AMODE, BMODE, EPIM>(L, st, dry) : launch_t<4, AMODE, BMODE, EPIM>(L, st, dry))

    if (type == MUCU_FWD && algo == MUCU_ALGO_IMPLICIT_GEMM && small_c_tc(g) && g.q <= 128 && g.k <= 256 &&
        env_int("MUCU_STAGED", 1)) {
        // Staged-row forward, zero workspace: tile = Tr whole output rows of
        // one image (Tr * Q <= 128 GEMM rows), K = the exact taps padded to whole k-blocks.
        const int Tr = 128 / g.q;
        const int num_kb = (int)ceil_div(RSC, KB);
        const int XR = g.stride * (Tr - 1) + g.r;
        const int WC = g.w * g.c;
        const int vec = 16 / elt;
        // TMA destinations 128-B aligned: a 128-B left margin (>= pad*C zero elements) and
        // rows of a multiple of 128 B
        (void)vec;
        const int xoff = (int)align_up((uint64_t)g.pad * g.c, (uint64_t)(128 / elt));
        const int SR = (int)align_up((uint64_t)(xoff + WC + g.pad * g.c), (uint64_t)(128 / elt));
        int cs = 0;
        for (int c = 256; c >= 1 && !cs; --c)
            if (WC % c == 0 && (c * elt) % 16 == 0 && WC / c <= 256) cs = c;
        const int BN = (int)align_up((uint64_t)g.k, 16);
        const int wbytes = (int)align_up((uint64_t)num_kb * BN * 128, 1024);
        const int sx_bytes = (int)align_up((uint64_t)XR * SR * elt, 1024);
        const int tabb = (int)align_up((uint64_t)num_kb * KB * 4, 1024);
        int Ss = 0, SX = 0;
        for (int sx : {2, 1})
            for (int sa : {4, 3, 2})
                if (!Ss && wbytes + sx * sx_bytes + tabb + sa * 16384 <= 222 * 1024) { Ss = sa; SX = sx; }
        if (cs && Ss && XR <= 256 && (WC * elt) % 16 == 0) {
            const int64_t tiles = (int64_t)b * ceil_div(g.p, Tr);
            A.M = (int)(tiles * 128); A.N = g.k; A.BN = BN; A.ldc = g.k; A.num_kb = num_kb; A.kred_taps = (int)RSC;
            A.mt = 1; A.km = 1; A.b_bytes = 0; A.bn_atoms = (BN * elt + 127) / 128;
            A.win_qb = Tr; A.sx_cs = xoff; A.sx_sr = SR; A.sx_tx = XR * WC * elt; A.sx_bytes = sx_bytes;
            A.sx_stages = SX; A.sxw_off = wbytes; A.bres_bytes = wbytes + SX * sx_bytes + tabb; A.stages = Ss;
            A.nacc = 2; A.tmem_cols = BN * 2 <= 64 ? 64 : BN * 2 <= 128 ? 128 : BN * 2 <= 256 ? 256 : 512;
            A.bsrc = in1;
            grid2(1);
            uint64_t dims[4] = {(uint64_t)cs, (uint64_t)(WC / cs), (uint64_t)g.h, (uint64_t)b};
            uint64_t str[3] = {(uint64_t)cs * elt, (uint64_t)WC * elt, (uint64_t)g.h * WC * elt};
            uint32_t box[4] = {(uint32_t)cs, (uint32_t)(WC / cs), 1, 1};
            if (!make_map(&L.ta, elt, in0, 4, dims, str, box, false, 0)) return -1;
            return LAUNCH(A_STAGED_FWD, B_RESIDENT, EPI_STORE);
        }
    }
    if (type == MUCU_FWD && algo == MUCU_ALGO_IMPLICIT_GEMM) {
        A.M = (int)(b * PQ); A.N = g.k; A.kred = (int)RSC; A.gsrc = in0;
        finalize_tiling(L, elt);
        grid2(1);
        A.ldc = g.k;
        const bool waligned = (RSC * elt) % 16 == 0;
        if (Aok) {
            A.num_kb = (int)ceil_div(RSC, KB);
            if (!waligned) return -1;
            if (!map2(&L.tb, in1, RSC, g.k, RSC, KB, A.BN)) return -1;
            if (g.stride == 1) {
                Launch H = L;
                H.a.mt = (H.a.BN <= 128 && env_int("MUCU_MT2", 1)) ? 2 : 1;
                size_stages(H.a);
                if (halo_setup(H.a, elt, b, g.p, g.q, g.r, g.s, g.pad, g.c)) {
                    uint64_t dims[4] = {(uint64_t)g.c, (uint64_t)g.w, (uint64_t)g.h, (uint64_t)b};
                    uint64_t str[3] = {(uint64_t)g.c * elt, (uint64_t)g.w * g.c * elt, (uint64_t)g.h * g.w * g.c * elt};
                    uint32_t box[4] = {(uint32_t)KB, (uint32_t)H.a.hx_W, 1, 1};
                    if (make_map(&H.ta, elt, in0, 4, dims, str, box)) {
                        L = H;
                        grid2(1);
                        A.tma_bytes = A.BN * 128;
                        return LAUNCH(A_HALO, B_TMA_K2, EPI_STORE);
                    }
                }
            }
            if (use_tma_im2col() &&
                im2col_a(elt, in0, g.c, g.w, g.h, b, -g.pad, -g.pad, g.pad - (g.s - 1),
                                g.pad - (g.r - 1), 128, g.stride, false)) {
                use_mt2(L, num_sms);
                grid2(1);
                A.tma_bytes = 16384 * A.mt + A.BN * 128;
                return LAUNCH(A_TMA_IM2COL, B_TMA_K2, EPI_STORE);
            }
            A.tma_bytes = A.BN * 128;
            err = LAUNCH(A_GATHER_FWD, B_TMA_K2, EPI_STORE);
        } else {
            A.bsrc = in1; A.ldb = (int)RSC;
            if (g.c * elt < 16) {
                // RGB-like layer: K' = (r, s8, c') with 8 taps x 16 B per k-block,
                // the zero-padded filter staged once per CTA in shared memory.
                A.cp = 16 / elt; A.s8 = (int)align_up((uint64_t)g.s, 8);
                A.num_kb = g.r * (A.s8 / 8);
                // The tap-group K layout (and with it the summation order) must not depend
                // on the micro-batch size (invariant I1): one N tile of exactly K columns,
                // whatever pick_bn's wave count would prefer at this b.
                if (g.k <= 256) {
                    A.BN = std::max(32, (int)align_up((uint64_t)g.k, 32));
                    A.bn_atoms = (A.BN * elt + 127) / 128;
                }
                if (ceil_div(A.N, A.BN) == 1) {
                    A.b_bytes = 0;
                    A.bres_bytes = A.num_kb * A.BN * 128;
                    A.stages = std::min(8, (kSmemBudget - A.bres_bytes) / (128 * 128));
                    if (A.stages >= 2) {
                        A.tma_bytes = 0;
                        return LAUNCH(A_GATHER_SMALLC, B_RESIDENT, EPI_STORE);
                    }
                }
                finalize_tiling(L, elt);
                A.cp = 0; A.s8 = 0; A.bres_bytes = 0;
            }
            A.num_kb = (int)ceil_div(RSC, KB);
            err = LAUNCH(A_SCALAR_FWD, B_SCALAR_K, EPI_STORE);
        }
        return err;
    }
    StagedWg zw_;
    if (algo == MUCU_ALGO_IM2COL_GEMM && win_tc(g, type) && !staged_wg_geom(g, &zw_)) {
        // Window WGRAD: dw^T[j][k] = sum over pixels of window(j, m) dy(m, k),
        // rows j = (r, atom, tap, c) over the padded copy xp, columns = the K filters.
        const Win z = win_geom(g);
        char* xp = ws + WL.a_off;
        err = DRY(launch_win_pad(g, b, z.Wp, in0, xp, st));
        if (err) return err;
        A.M = z.M; A.N = g.k; A.ldc = RSC; A.kred = (int)(b * PQ); A.cp = z.cpx; A.win_na = z.na; A.win_aw = z.aw;
        wgrad_tiling(atom, true, g.q);
        const int KD = KB * A.km;
        const uint64_t pb = (uint64_t)z.cpx * elt;
        const int wat = z.aw / elt;  // elements per A atom
        // One 5-D box per 128-row half when the half holds whole filter rows: view
        // {atom element, output pixel q (stride st*16 B), atom aa, input row h, image}
        // gives the smem order [r][aa][q][element] the per-atom boxes produce, in one
        // TMA instead of 4-8 small ones (filter rows past R load real data, discarded).
        const int atoms_half = 128 * elt / z.aw;
        if (atoms_half % z.na == 0 && env_int("MUCU_WIN_BOX", 1)) {
            const int hext = atoms_half / z.na;
            uint64_t adims[5] = {(uint64_t)wat, (uint64_t)g.q, (uint64_t)z.na, (uint64_t)g.h, (uint64_t)b};
            uint64_t astr[4] = {g.stride * pb, (uint64_t)wat * elt, z.Wp * pb, (uint64_t)g.h * z.Wp * pb};
            uint32_t abox[5] = {(uint32_t)wat, (uint32_t)KD, (uint32_t)z.na, (uint32_t)hext, 1};
            if (make_map(&L.ta, elt, xp, 5, adims, astr, abox, true, z.aw)) A.win_box = hext;
        }
        if (!A.win_box) {
            uint64_t adims[4] = {(uint64_t)z.na * wat, (uint64_t)g.q, (uint64_t)g.h, (uint64_t)b};
            uint64_t astr[3] = {g.stride * pb, z.Wp * pb, (uint64_t)g.h * z.Wp * pb};
            uint32_t abox[4] = {(uint32_t)wat, (uint32_t)KD, 1, 1};
            if (!make_map(&L.ta, elt, xp, 4, adims, astr, abox, true, z.aw)) return -1;
        }
        if (!map3(&L.tb, in1, g.k, g.q, (uint64_t)b * g.p, g.k, (uint64_t)g.q * g.k, atom, KD, 1, true)) return -1;
        A.tma_bytes = A.km * (A.mt * 128 * KB * elt + A.bn_atoms * KB * 128);
        if (ctx->deterministic) {
            // Deterministic split-K through the workspace: one split per SM
            // (at most kPartialSlots) writes its partial tile [z.M rows][K] fp32; a reduction
            // kernel sums the slots in split order and scatters the window rows into dw --
            // every SM busy, no cluster packing loss or ordered group hand-offs.
            const int64_t nkb = (int64_t)b * g.p * A.win_qb;
            const int64_t S = std::max<int64_t>(1, std::min<int64_t>(std::min<int64_t>(kPartialSlots, num_sms), nkb));
            A.num_kb = (int)nkb;
            A.kb_per_split = (int)ceil_div(nkb, S);
            const int64_t Sr = ceil_div(nkb, A.kb_per_split);
            A.cl = 0; A.zsplit = 0; A.atomic = 0; A.stg_bytes = 0;
            A.num_z = (int)Sr;
            L.grid = dim3((unsigned)Sr);
            float* part = (float*)(ws + WL.b_off);
            A.out = part; A.alpha = 1.f; A.beta = 0.f; A.ldc = g.k; A.part_rows = z.M;
            if (z.aw == 64) err = LAUNCH(A_TMA_WIN64, B_TMA_DYROW, EPI_WGRAD_PARTIAL);
            else if (z.aw == 32) err = LAUNCH(A_TMA_WIN32, B_TMA_DYROW, EPI_WGRAD_PARTIAL);
            else err = LAUNCH(A_TMA_WIN, B_TMA_DYROW, EPI_WGRAD_PARTIAL);
            if (err) return err;
            note_fused();
            return DRY(launch_partial_reduce_win((int)Sr, (int64_t)z.M * g.k, z.M, g.k, z.aw / elt, z.cpx, z.na, g,
                                                 part, alpha, beta, (float*)out, st, mc_reduce));
        }
        if (z.aw == 64) return LAUNCH(A_TMA_WIN64, B_TMA_DYROW, EPI_WGRAD_WIN);
        if (z.aw == 32) return LAUNCH(A_TMA_WIN32, B_TMA_DYROW, EPI_WGRAD_WIN);
        return LAUNCH(A_TMA_WIN, B_TMA_DYROW, EPI_WGRAD_WIN);
    }
    if (algo == MUCU_ALGO_IM2COL_GEMM && s2d_tc(g, type) && !(type == MUCU_BWD_FILTER && staged_wg_geom(g, &zw_))) {
        // Space-to-depth: the strided small-C layer as a stride-1
        // Dr x Ds conv over the super-pixel image with Cs channels -- 128-B
        // channel atoms, so TMA im2col feeds it like any other layer.
        const S2d z = s2d_geom(g, type);
        const int st_ = g.stride, Dr = z.Dr, Ds = z.Ds, Cs = z.Cs;
        const int kind = type == MUCU_BWD_DATA ? 4 : 3;
        if (type != MUCU_BWD_FILTER && (ctx->fixed_kind != kind || ctx->fixed_src != in1)) {
            err = DRY(launch_s2d_filter(g, type == MUCU_BWD_DATA, z, in1, ws, st));
            if (err) return err;
            ctx->fixed_kind = kind; ctx->fixed_src = in1;
        }
        A.s2_st = st_; A.s2_C = g.c; A.s2_R = g.r; A.s2_S = g.s;
        if (type == MUCU_BWD_DATA) {
            // dx in f x f super-pixels (f = st*u, s2d_geom): super-pixel (i, j) takes dy
            // pixels (u*i + u-1-d, u*j + u-1-e), d < Dr, e < Ds -- a TMA im2col walk with
            // traversal stride u and flipped taps; the depth-to-space epilogue writes
            // dx[n][f*i + a' - pad][f*j + b' - pad][c] for column (a', b', c).
            const int I = z.I, J = z.J, f = z.f, u = z.u;
            const int Kp = Dr * Ds * g.k;
            A.s2_st = f;
            A.M = b * I * J; A.N = f * f * g.c; A.num_kb = Kp / KB; A.kred = Kp;
            A.ph_mode = 1; A.ph_H = I; A.ph_W = J; A.ph_i0 = 0; A.ph_j0 = 0;
            A.tapR = Dr; A.tapS = Ds; A.im2col_dgrad = 1; A.gsrc = in0; A.ph_u = u;
            A.e_H = g.h; A.e_W = g.w; A.e_C = g.c; A.e_pad = g.pad;
            finalize_tiling(L, elt);
            // The row-wise depth-to-space epilogue reads TMEM in 4-column pieces, so the
            // tile can be exactly N = f*f*C columns when that is a legal UMMA N (ResNet:
            // 48 instead of 64)
            const bool rows_ok = beta == 0.f && (f * g.c) % 4 == 0 && env_int("MUCU_D2S_ROWS", 1);
            if (rows_ok && A.N < A.BN && A.N % 16 == 0 && env_int("MUCU_D2S_EXACT_N", 1)) {
                A.BN = A.N;
                A.bn_atoms = (A.BN * elt + 127) / 128;
                A.b_bytes = std::max(A.BN * 128, A.bn_atoms * (128 / elt) * 128);
                size_stages(A);
            }
            use_mt2(L, num_sms);
            grid2(1);
            // start pixel of super-pixel (i, j): (u*i - (Dr - u), u*j - (Ds - u)); the kernel's
            // phase-mode origin is ph_i0 + ii - (tapR - 1) in map units, so the map walks u-strided
            // positions lw, lw + u, ... with J of them per row.
            const int lw = -(Ds - u), lh = -(Dr - u);
            if (!im2col_a(elt, in0, g.k, g.q, g.p, b, lw, lh, lw + u * (J - 1) - (g.q - 1),
                                 lh + u * (I - 1) - (g.p - 1), 128, u, false))
                return -1;
            if (!map2(&L.tb, ws, Kp, A.N, Kp, KB, A.BN)) return -1;
            A.tma_bytes = 16384 * A.mt + A.BN * 128;
            A.d2s_rows = rows_ok && A.N <= A.BN;
            return LAUNCH(A_TMA_IM2COL, B_TMA_K2, EPI_D2S);
        }
        const int I = z.I, J = z.J;
        char* xs = ws + WL.a_off;
        err = DRY(launch_s2d_input(g, b, z.f, I, J, Cs, in0, xs, st));
        if (err) return err;
        // the GEMM sees the stride-1, pad-0 geometry over xs (Pu x Qu output super-pixels)
        A.H = I; A.W = J; A.C = Cs; A.R = Dr; A.S = Ds; A.pad = 0; A.stride = 1; A.tapR = Dr; A.tapS = Ds;
        A.P = z.Pu; A.Q = z.Qu;
        if (type == MUCU_FWD) {
            const int Kp = Dr * Ds * Cs;
            A.M = b * z.Pu * z.Qu; A.N = z.u * z.u * g.k; A.ldc = g.k; A.num_kb = Kp / KB; A.kred = Kp;
            A.gsrc = xs;
            finalize_tiling(L, elt);
            use_mt2(L, num_sms);
            grid2(1);
            if (!im2col_a(elt, xs, Cs, J, I, b, 0, 0, -(Ds - 1), -(Dr - 1), 128, 1, false)) return -1;
            if (!map2(&L.tb, ws, Kp, A.N, Kp, KB, A.BN)) return -1;
            A.tma_bytes = 16384 * A.mt + A.BN * 128;
            if (z.u == 1) return LAUNCH(A_TMA_IM2COL, B_TMA_K2, EPI_STORE);
            // u x u output super-pixels: column (uu, vv, k) -> y[n][u*i' + uu][u*j' + vv][k]
            A.ph_H = z.Pu; A.ph_W = z.Qu; A.s2_st = z.u;
            A.e_H = g.p; A.e_W = g.q; A.e_C = g.k; A.e_pad = 0;
            return LAUNCH(A_TMA_IM2COL, B_TMA_K2, EPI_D2S);
        }
        // WGRAD (u = 1): dw'[k][(d, e, c')] = sum_m dy[m][k] xs(m; d, e, c'), folded
        // into dw[k][st*d + a][st*e + b][c] by the epilogue's reductions.
        const int64_t Mpix = (int64_t)b * PQ;
        A.M = g.k; A.N = Dr * Ds * Cs; A.ldc = RSC; A.kred = (int)Mpix; A.gsrc = xs;
        wgrad_tiling(atom, true);
        if (!map2(&L.ta, in1, g.k, (uint64_t)Mpix, g.k, atom, KB * A.km, true)) return -1;
        if (!make_im2col_map(&L.tb, elt, xs, Cs, J, I, b, 0, 0, -(Ds - 1), -(Dr - 1), KB * A.km, 1, true))
            return -1;
        A.tma_bytes = A.km * (A.mt * 128 * KB * elt + A.bn_atoms * KB * 128);
        return LAUNCH(A_TMA_MN2, B_TMA_IM2COL, EPI_WGRAD_S2D);
    }
    if (type == MUCU_FWD && algo == MUCU_ALGO_IM2COL_GEMM && small_c_tc(g)) {
        // RGB-like layer: x -> channel-padded copy (16 B / pixel) in the workspace,
        // then the tap-walking GEMM with async 16-B gathers and the staged filter.
        err = DRY(launch_pad_channels(g, b, in0, ws + WL.a_off, st));
        if (err) return err;
        A.M = (int)(b * PQ); A.N = g.k; A.ldc = g.k; A.gsrc = ws + WL.a_off; A.bsrc = in1;
        A.cp = 16 / elt; A.s8 = (int)align_up((uint64_t)g.s, 8);
        A.num_kb = g.r * (A.s8 / 8);
        finalize_tiling(L, elt);
        if (ceil_div(A.N, A.BN) != 1) return -1;
        A.b_bytes = 0;
        A.bres_bytes = A.num_kb * A.BN * 128;
        A.stages = std::min(8, (kSmemBudget - A.bres_bytes) / (128 * 128));
        if (A.stages < 2) return -1;
        grid2(1);
        A.tma_bytes = 0;
        return LAUNCH(A_GATHER_SMALLC_PAD, B_RESIDENT, EPI_STORE);
    }
    if (type == MUCU_FWD && algo == MUCU_ALGO_IM2COL_GEMM) {
        const void* colp = in0;
        int kpitch = g.c;
        if (!is_pointwise(g)) {
            colp = ws + WL.a_off;
            kpitch = WL.kpitch;
            err = DRY(launch_im2col(g, b, in0, (void*)colp, kpitch, st));
            if (err) return err;
        }
        const void* wp = in1;
        int wpitch = (int)RSC;
        if (WL.filter_padded) {
            if (ctx->fixed_kind != 1 || ctx->fixed_src != in1) {
                err = DRY(launch_pad_filter(g, in1, ws, WL.kpitch, st));
                if (err) return err;
                ctx->fixed_kind = 1; ctx->fixed_src = in1;
            }
            wp = ws; wpitch = WL.kpitch;
        }
        A.M = (int)(b * PQ); A.N = g.k; A.num_kb = (int)ceil_div(RSC, KB); A.ldc = g.k;
        finalize_tiling(L, elt);
        use_mt2(L, num_sms);
        grid2(1);
        if (!map2(&L.ta, colp, RSC, (uint64_t)A.M, kpitch, KB, 128)) return -1;
        if (!map2(&L.tb, wp, RSC, g.k, wpitch, KB, A.BN)) return -1;
        A.tma_bytes = 16384 * A.mt + A.BN * 128;
        return LAUNCH(A_TMA_K2, B_TMA_K2, EPI_STORE);
    }
    if (algo == MUCU_ALGO_WINOGRAD_2X2_3X3 && type == MUCU_BWD_FILTER) {
        // Winograd F(3x3,2x2) BackwardFilter: transforms, then 16 GEMMs
        // M_xi[k][c] = sum_t D_xi[t][k] V_xi[t][c] as one batched split-K launch
        // (z = xi * splits + split, fp32 reductions into the zeroed M), then
        // dw = alpha * G^T M G + beta * dw.
        const int Cp = (int)align_up((uint64_t)g.c, (uint64_t)atom), Kp = (int)align_up((uint64_t)g.k, (uint64_t)atom);
        const int64_t Tp = (int64_t)align_up((uint64_t)b * ((g.p + 1) / 2) * ((g.q + 1) / 2), 256);
        if (16 * Tp > INT32_MAX) return -1;
        void* V = ws + WL.a_off;
        void* D = ws + WL.b_off;
        float* Mx = (float*)(ws + WL.fixed_off);
        err = DRY(launch_wgw_transforms(g, b, in0, in1, V, D, Tp, st));
        if (err) return err;
        A.M = g.k; A.N = g.c; A.ldc = Cp; A.kred = (int)Tp; A.out = Mx; A.alpha = 1.f; A.beta = 0.f; A.out_bf16 = 0;
        A.batch_stride = (long long)Kp * Cp;
        wgrad_tiling(16, true, 0, 4, 16);
        if (!A.zsplit) A.zsplit = 1;  // batch = z / zsplit (one split per batch)
        A.zrows = (int)Tp;
        if (!map2(&L.ta, D, Kp, 16 * Tp, Kp, atom, KB * A.km, true)) return -1;
        if (!map2(&L.tb, V, Cp, 16 * Tp, Cp, atom, KB * A.km, true)) return -1;
        map_mn_box(V, Cp, 16 * Tp, Cp, KB * A.km);
        A.tma_bytes = A.km * (A.mt * 128 * KB * elt + A.bn_atoms * KB * 128);
        err = LAUNCH(A_TMA_MN2, B_TMA_MN2, EPI_WGRAD_CHAIN);
        if (err) return err;
        return DRY(launch_wgw_output(g, alpha, Mx, beta, (float*)out, st));
    }
    if (algo == MUCU_ALGO_WINOGRAD_2X2_3X3) {
        const bool dg = type == MUCU_BWD_DATA;
        const int I = dg ? g.k : g.c, O = dg ? g.c : g.k;
        const int OH = dg ? g.h : g.p, OW = dg ? g.w : g.q;
        const int64_t Tt = (int64_t)((OH + 1) / 2) * ((OW + 1) / 2) * b;
        if (ctx->fixed_kind != 2 || ctx->fixed_src != in1) {
            err = DRY(launch_wg_filter(g, dg, in1, ws, st));
            if (err) return err;
            ctx->fixed_kind = 2; ctx->fixed_src = in1;
        }
        void* V = ws + WL.a_off;
        float* Mx = (float*)(ws + WL.b_off);
        err = DRY(launch_wg_input(g, dg, b, in0, V, st));
        if (err) return err;
        A.M = (int)Tt; A.N = O; A.num_kb = (int)ceil_div(I, KB); A.ldc = O;
        A.batch_stride = Tt * O; A.alpha = 1.f; A.beta = 0.f; A.out = Mx; A.out_bf16 = 0;
        finalize_tiling(L, elt, 32, 16);
        grid2(16);
        if (!map3(&L.ta, V, I, Tt, 16, I, Tt * I, KB, 128, 1)) return -1;
        if (!map3(&L.tb, ws, I, O, 16, I, (uint64_t)O * I, KB, A.BN, 1)) return -1;
        A.tma_bytes = 16384 * A.mt + A.BN * 128;
        err = LAUNCH(A_TMA_K3, B_TMA_K3, EPI_STORE);
        if (err) return err;
        return DRY(launch_wg_output(g, dg, b, alpha, Mx, beta, out, st));
    }
    if (type == MUCU_BWD_DATA && algo == MUCU_ALGO_IMPLICIT_GEMM && g.c <= 4 && env_int("MUCU_SMALLC_DGRAD", 1)) {
        // RGB layer: N = C <= 4 output columns fit no tensor-core tile; zero-workspace
        // FFMA kernel over the phase sub-filters (kernels_simt.cu small_c_dgrad)
        if (dry) return 0;
        const int e = small_c_dgrad(g, b, alpha, in0, in1, beta, out, st);
        if (e != -1) return e;
    }
    if (type == MUCU_BWD_DATA && algo == MUCU_ALGO_IMPLICIT_GEMM && g.stride > 1 && g.k % KB == 0 &&
        use_tma_im2col()) {
        // Strided DGRAD by phase decomposition: one stride-1 transposed conv per
        // phase (r0, s0) over the dx sub-grid it owns, with only its
        // ceil((R-r0)/st) x ceil((S-s0)/st) taps -- no masked (zero) taps.
        const bool bvec = (g.c * elt) % 16 == 0 && g.c >= atom;
        if (bvec && !map3(&L.tb, in1, g.c, RS, g.k, g.c, RSC, atom, 1, KB, true)) return -1;
        A.gsrc = in0; A.bsrc = in1; A.ldc = g.c; A.N = g.c;
        A.ph_mode = 1; A.im2col_dgrad = 1;
        finalize_tiling(L, elt);
        // beta = 0: the phases that meet no tap (r0 >= R or s0 >= S) are zeroed in one
        // elementwise pass instead of one GEMM launch each
        const bool zero_pass = beta == 0.f && (g.r < g.stride || g.s < g.stride) && (g.c * elt) % 16 == 0;
        if (zero_pass) {
            err = DRY(launch_zero_tapless(g, b, out, st));
            if (err) return err;
        }
        // One launch for all phases with taps when they tile equal sub-grids whose
        // dy start pixels share one im2col map (equal lower corners i0 - (nr-1),
        // j0 - (ns-1)); tiles of phase z are blockIdx-tiles of batch z.
        if (bvec && env_int("MUCU_MERGE_PHASES", 1) && g.stride * g.stride <= 4) {
            int n_ph = 0, H0 = -1, W0 = -1, lh0 = 0, lw0 = 0;
            bool ok = true;
            for (int r0 = 0; r0 < g.stride && ok; ++r0) {
                for (int s0 = 0; s0 < g.stride && ok; ++s0) {
                    const int i0 = std::max(0, (int)ceil_div(g.pad - r0, g.stride));
                    const int j0 = std::max(0, (int)ceil_div(g.pad - s0, g.stride));
                    const int hb = r0 - g.pad + g.stride * i0, wb = s0 - g.pad + g.stride * j0;
                    const int Hph = hb < g.h ? (int)ceil_div(g.h - hb, g.stride) : 0;
                    const int Wph = wb < g.w ? (int)ceil_div(g.w - wb, g.stride) : 0;
                    const int nr = r0 < g.r ? (int)ceil_div(g.r - r0, g.stride) : 0;
                    const int ns = s0 < g.s ? (int)ceil_div(g.s - s0, g.stride) : 0;
                    if (Hph <= 0 || Wph <= 0) continue;
                    if (nr == 0 || ns == 0) { ok = zero_pass; continue; }
                    const int lh = i0 - (nr - 1), lw = j0 - (ns - 1);
                    if (n_ph == 0) { H0 = Hph; W0 = Wph; lh0 = lh; lw0 = lw; }
                    ok = Hph == H0 && Wph == W0 && lh == lh0 && lw == lw0;
                    A.ph_r0v[n_ph] = r0; A.ph_s0v[n_ph] = s0; A.ph_i0v[n_ph] = i0; A.ph_j0v[n_ph] = j0;
                    A.ph_hbv[n_ph] = hb; A.ph_wbv[n_ph] = wb; A.ph_tRv[n_ph] = nr; A.ph_tSv[n_ph] = ns;
                    A.ph_kbv[n_ph] = nr * ns * (g.k / KB);
                    ++n_ph;
                }
            }
            if (ok && n_ph > 1) {
                A.ph_n = n_ph; A.ph_H = H0; A.ph_W = W0;
                A.tapR = A.ph_tRv[0]; A.tapS = A.ph_tSv[0];
                A.M = b * H0 * W0;
                A.num_kb = 0;
                for (int z = 0; z < n_ph; ++z) A.num_kb = std::max(A.num_kb, A.ph_kbv[z]);
                if (!im2col_a(elt, in0, g.k, g.q, g.p, b, lw0, lh0, lw0 + W0 - g.q, lh0 + H0 - g.p, 128,
                                     1, false))
                    return -1;
                A.mt = 1;
                size_stages(A);
                // 512-/256-row tiles only when every phase alone has a tile per SM
                use_mt2(L, num_sms);
                grid2(n_ph);
                A.tma_bytes = 16384 * A.mt + A.bn_atoms * KB * 128;
                map_w_box(in1);
                return LAUNCH(A_TMA_IM2COL, B_TMA_MN3, EPI_STORE);
            }
            A.ph_n = 0;
        }
        for (int r0 = 0; r0 < g.stride; ++r0) {
            for (int s0 = 0; s0 < g.stride; ++s0) {
                // dx rows with (h + pad) % st == r0: h = r0 - pad + st*i, i >= i0
                const int i0 = std::max(0, (int)ceil_div(g.pad - r0, g.stride));
                const int j0 = std::max(0, (int)ceil_div(g.pad - s0, g.stride));
                const int hb = r0 - g.pad + g.stride * i0, wb = s0 - g.pad + g.stride * j0;
                const int Hph = hb < g.h ? (int)ceil_div(g.h - hb, g.stride) : 0;
                const int Wph = wb < g.w ? (int)ceil_div(g.w - wb, g.stride) : 0;
                if (Hph <= 0 || Wph <= 0) continue;
                const int nr = r0 < g.r ? (int)ceil_div(g.r - r0, g.stride) : 0;
                const int ns = s0 < g.s ? (int)ceil_div(g.s - s0, g.stride) : 0;
                if (zero_pass && (nr == 0 || ns == 0)) continue;
                A.ph_H = Hph; A.ph_W = Wph; A.ph_i0 = i0; A.ph_j0 = j0; A.ph_r0 = r0; A.ph_s0 = s0;
                A.ph_hb = hb; A.ph_wb = wb; A.tapR = std::max(nr, 1); A.tapS = std::max(ns, 1);
                A.M = b * Hph * Wph;
                A.num_kb = (nr > 0 && ns > 0) ? nr * ns * (g.k / KB) : 0;  // 0 taps: dx = beta * dx
                A.kred = nr * ns * g.k;
                grid2(1);
                // dy im2col: start positions i0 - (nr-1) ... (Hph of them), stride 1
                const int lh = i0 - (A.tapR - 1), lw = j0 - (A.tapS - 1);
                if (A.num_kb > 0 &&
                    !im2col_a(elt, in0, g.k, g.q, g.p, b, lw, lh, lw + Wph - g.q, lh + Hph - g.p,
                                     128, 1, false))
                    return -1;
                A.mt = 1;
                size_stages(A);
                use_mt2(L, num_sms);
                grid2(1);
                A.tma_bytes = 16384 * A.mt + (bvec ? A.bn_atoms * KB * 128 : 0);
                if (bvec) map_w_box(in1);
                err = bvec ? LAUNCH(A_TMA_IM2COL, B_TMA_MN3, EPI_STORE) : LAUNCH(A_TMA_IM2COL, B_SCALAR_DGRAD, EPI_STORE);
                if (err) return err;
            }
        }
        return 0;
    }
    if (type == MUCU_BWD_DATA && algo == MUCU_ALGO_IMPLICIT_GEMM) {
        A.M = (int)(b * HW); A.N = g.c; A.num_kb = (int)ceil_div((int64_t)RS * g.k, KB); A.ldc = g.c;
        A.gsrc = in0; A.kred = RS * g.k;
        finalize_tiling(L, elt);
        grid2(1);
        A.bsrc = in1;
        if (g.k % KB != 0) return LAUNCH(A_SCALAR_DGRAD, B_SCALAR_DGRAD, EPI_STORE);
        if ((g.c * elt) % 16 == 0 && g.c >= atom) {
            // w viewed as {C, R*S, K} (c contiguous): B(c, (r,s,k)) MN-major
            if (!map3(&L.tb, in1, g.c, RS, g.k, g.c, RSC, atom, 1, KB, true)) return -1;
            if (g.stride == 1 && g.pad <= g.r - 1 && g.pad <= g.s - 1) {
                // transposed conv = correlation of dy with the flipped filter, origin R-1-pad
                Launch H = L;
                if (g.c > 128 && g.c % 128 == 0 && !env_int("MUCU_FORCE_BN", 0)) H.a.BN = 128;
                H.a.bn_atoms = (H.a.BN * elt + 127) / 128;
                H.a.b_bytes = std::max(H.a.BN * 128, H.a.bn_atoms * (128 / elt) * 128);
                H.a.mt = (H.a.BN <= 128 && env_int("MUCU_MT2", 1)) ? 2 : 1;
                size_stages(H.a);
                if (g.r - 1 - g.pad == g.s - 1 - g.pad &&
                    halo_setup(H.a, elt, b, g.h, g.w, g.r, g.s, g.r - 1 - g.pad, g.k)) {
                    uint64_t dims[4] = {(uint64_t)g.k, (uint64_t)g.q, (uint64_t)g.p, (uint64_t)b};
                    uint64_t str[3] = {(uint64_t)g.k * elt, (uint64_t)g.q * g.k * elt, (uint64_t)g.p * g.q * g.k * elt};
                    uint32_t box[4] = {(uint32_t)KB, (uint32_t)H.a.hx_W, 1, 1};
                    if (make_map(&H.ta, elt, in0, 4, dims, str, box)) {
                        L = H;
                        grid2(1);
                        A.tma_bytes = A.bn_atoms * KB * 128;
                        return LAUNCH(A_HALO, B_TMA_MN3, EPI_STORE);
                    }
                }
            }
            // stride 1: im2col of dy with pad' = R-1-pad and flipped taps
            const int lw = g.pad - (g.s - 1), lh = g.pad - (g.r - 1);
            if (g.stride == 1 && use_tma_im2col() &&
                im2col_a(elt, in0, g.k, g.q, g.p, b, lw, lh, lw + g.w - g.q, lh + g.h - g.p, 128, 1,
                                false)) {
                A.im2col_dgrad = 1;
                // C a multiple of 128 (> 128): 256 x 128 tiles (two interleaved
                // accumulators) beat 128 x min(C, 256) ones (measured, AlexNet conv4/5)
                if (g.c > 128 && g.c % 128 == 0 && ceil_div(A.M, 256) >= num_sms && !env_int("MUCU_FORCE_BN", 0)) {
                    A.BN = 128;
                    A.bn_atoms = (A.BN * elt + 127) / 128;
                    A.b_bytes = std::max(A.BN * 128, A.bn_atoms * (128 / elt) * 128);
                    size_stages(A);
                }
                use_mt2(L, num_sms);
                grid2(1);
                A.tma_bytes = 16384 * A.mt + A.bn_atoms * KB * 128;
                map_w_box(in1);
                return LAUNCH(A_TMA_IM2COL, B_TMA_MN3, EPI_STORE);
            }
            A.tma_bytes = A.bn_atoms * KB * 128;
            return LAUNCH(A_GATHER_DGRAD, B_TMA_MN3, EPI_STORE);
        }
        return LAUNCH(A_GATHER_DGRAD, B_SCALAR_DGRAD, EPI_STORE);
    }
    if (type == MUCU_BWD_DATA && algo == MUCU_ALGO_IM2COL_GEMM) {
        // dcol[m', (r,s,c)] = sum_k dy[m'][k] w[k][(r,s,c)]  (pointwise: straight into dx with alpha/beta)
        const bool pw = is_pointwise(g);
        const void* wp = in1;
        int64_t wpitch = RSC;
        if (!pw && WL.filter_padded) {
            // same pitch as ws_layout: one 128-B atom for short rows, else 16 B
            const int fpitch = RSC < atom ? atom : (int)align_up((uint64_t)RSC, (uint64_t)(16 / elt));
            if (ctx->fixed_kind != 1 || ctx->fixed_src != in1) {
                err = DRY(launch_pad_filter(g, in1, ws, fpitch, st));
                if (err) return err;
                ctx->fixed_kind = 1; ctx->fixed_src = in1;
            }
            wp = ws; wpitch = fpitch;
        }
        A.M = (int)(b * PQ); A.N = (int)RSC; A.num_kb = (int)ceil_div(g.k, KB);
        if (pw) { A.ldc = g.c; }
        else { A.ldc = WL.kpitch; A.out = ws + WL.a_off; A.out_bf16 = 0; A.alpha = 1.f; A.beta = 0.f; }
        finalize_tiling(L, elt);
        use_mt2(L, num_sms);
        grid2(1);
        if (wpitch < atom) return -1;  // pointwise with C < one atom
        if (!map2(&L.ta, in0, g.k, (uint64_t)A.M, g.k, KB, 128)) return -1;
        if (!map2(&L.tb, wp, std::max<int64_t>(RSC, atom), g.k, wpitch, atom, KB, true)) return -1;
        map_mn_box(wp, (uint64_t)std::max<int64_t>(RSC, atom), g.k, wpitch, KB);
        A.tma_bytes = 16384 * A.mt + A.bn_atoms * KB * 128;
        err = LAUNCH(A_TMA_K2, B_TMA_MN2, EPI_STORE);
        if (err || pw) return err;
        return DRY(launch_col2im(g, b, alpha, (const float*)(ws + WL.a_off), WL.kpitch, beta, out, st));
    }
    if (type == MUCU_BWD_FILTER) {
        // dw[k][(r,s,c)] = sum_m dy[m][k] B(m, (r,s,c)); A = dy MN-major via TMA.
        const int64_t Mpix = (int64_t)b * PQ;
        A.M = g.k; A.N = (int)RSC; A.ldc = RSC; A.kred = (int)Mpix; A.gsrc = in0;
        // P:L58 output scale: split 0 of every tile applies the user's beta, later
        // splits add in split order (ordered turn counters, deterministic).
        const int a_bytes = 128 * KB * elt;
        // dy as the MN-major A operand: with K a multiple of the 128-B atom, a 3-D view
        // {atom element, pixel, atom index} loads a whole 128-row half (4 tf32 / 2 bf16
        // atoms) in one TMA box instead of one box per atom (AlexNet TF32 WGRAD -4..11 %,
        // BF16 IG WGRAD -3..5 %, pointwise within noise).
        auto map_dy = [&]() {
            A.a_box = 0;
            if (g.k % atom == 0 && env_int("MUCU_A_BOX", 1)) {
                uint64_t dims[3] = {(uint64_t)atom, (uint64_t)Mpix, (uint64_t)(g.k / atom)};
                uint64_t str[2] = {(uint64_t)g.k * elt, 128};
                uint32_t box[3] = {(uint32_t)atom, (uint32_t)(KB * A.km), (uint32_t)elt};
                if (make_map(&L.ta, elt, in1, 3, dims, str, box, true)) { A.a_box = 1; return true; }
            }
            return map2(&L.ta, in1, g.k, (uint64_t)Mpix, g.k, atom, KB * A.km, true);
        };
        StagedWg zw;
        if (((algo == MUCU_ALGO_IMPLICIT_GEMM && env_int("MUCU_STAGED", 1)) || algo == MUCU_ALGO_IM2COL_GEMM) &&
            staged_wg_geom(g, &zw)) {
            // Staged-row BackwardFilter: GEMM rows = the exact R*S*C taps
            // (padded only to 128-row halves), columns = the K filters, reduction = output
            // pixels in blocks of KD of one output row.  IG (zero workspace): cluster
            // split-K (6.9).  I2C: every split writes its partial tile to the workspace and
            // a reduction kernel sums them in split order.
            A.M = (int)RSC; A.N = g.k; A.ldc = (int)RSC; A.kred_taps = (int)RSC; A.mt = zw.mt; A.BN = g.k;
            A.bn_atoms = g.k * elt / 128; A.b_bytes = zw.b_bytes; A.km = 1;
            A.win_qb = (int)ceil_div(g.q, KB);
            A.sx_cs = zw.cs; A.sx_sr = zw.bch * zw.cs; A.sx_tx = zw.sx_tx; A.sx_bytes = zw.sx_bytes;
            A.stages = zw.Ss; A.sx_stages = zw.SX; A.bres_bytes = zw.SX * zw.sx_bytes + zw.tab_bytes;
            A.nacc = zw.mt * A.BN <= 256 ? 2 : 1;
            const int cols = A.nacc * zw.mt * A.BN;
            A.tmem_cols = cols <= 64 ? 64 : cols <= 128 ? 128 : cols <= 256 ? 256 : 512;
            const int64_t nkb = (int64_t)b * g.p * A.win_qb;
            const int WC = g.w * g.c;
            uint64_t dims[4] = {(uint64_t)zw.cs, (uint64_t)(WC / zw.cs), (uint64_t)g.h, (uint64_t)b};
            uint64_t str[3] = {(uint64_t)zw.cs * elt, (uint64_t)WC * elt, (uint64_t)g.h * WC * elt};
            uint32_t box[4] = {(uint32_t)zw.cs, (uint32_t)zw.bch, (uint32_t)g.r, 1};
            if (!make_map(&L.ta, elt, in0, 4, dims, str, box, false, 0)) return -1;
            if (!map3(&L.tb, in1, g.k, g.q, (uint64_t)b * g.p, g.k, (uint64_t)g.q * g.k, atom, KB, 1, true))
                return -1;
            A.tma_bytes = A.bn_atoms * KB * 128;
            if (algo == MUCU_ALGO_IMPLICIT_GEMM) {
                apply_split(1, nkb, 1, true);  // builders double as epilogue: one unit per CTA
                return LAUNCH(A_STAGED_WG, B_TMA_DYROW, EPI_WGRAD_TAPS);
            }
            // I2C: one split per SM (at most kPartialSlots), partial tiles [split][TR][BN] fp32
            const int64_t S = std::max<int64_t>(1, std::min<int64_t>(std::min<int64_t>(kPartialSlots, num_sms), nkb));
            A.num_kb = (int)nkb;
            A.kb_per_split = (int)ceil_div(nkb, S);
            const int64_t Sr = ceil_div(nkb, A.kb_per_split);
            A.cl = 0; A.zsplit = 0; A.atomic = 0; A.stg_bytes = 0;
            A.num_z = (int)Sr;
            L.grid = dim3((unsigned)Sr);
            float* part = (float*)(ws + WL.a_off);
            A.out = part; A.alpha = 1.f; A.beta = 0.f; A.ldc = g.k; A.part_rows = zw.TR;
            err = LAUNCH(A_STAGED_WG, B_TMA_DYROW, EPI_WGRAD_PARTIAL);
            if (err) return err;
            note_fused();
            return DRY(launch_partial_reduce((int)Sr, (int64_t)zw.TR * g.k, g.k, (int)RSC, g.k, true, part, alpha, beta,
                                             (float*)out, st, mc_reduce));
        }
        if (algo == MUCU_ALGO_IM2COL_GEMM && small_c_tc(g)) {
            // RGB-like layer: channel-padded copy of x, padded columns j' = (r, s8, c').
            err = DRY(launch_pad_channels(g, b, in0, ws + WL.a_off, st));
            if (err) return err;
            A.gsrc = ws + WL.a_off;
            A.cp = 16 / elt; A.s8 = (int)align_up((uint64_t)g.s, 8);
            A.N = g.r * A.s8 * A.cp;
            wgrad_tiling(atom, false);
            if (!map_dy()) return -1;
            A.tma_bytes = a_bytes;
            return LAUNCH(A_TMA_MN2, B_GATHER_SMALLC_PAD, EPI_WGRAD_SMALLC);
        }
        // Workspace partials: persistent CTAs over all SMs, split s writes its dW tile to
        // slot s, a reduction kernel sums the slots in order (no cluster packing loss, no
        // ordered hand-over).  `launch_partial(launch)` runs the GEMM launcher given.
        auto launch_partial = [&](const int P, auto launch) -> int {
            const int64_t tiles = ceil_div(A.N, A.BN) * ceil_div(A.M, 128 * A.mt);
            const int64_t nkb = A.num_kb;
            const double E = env_int("MUCU_SPLIT_E", 16) / (double)A.km;
            int64_t sbest = 1;
            double best = 1e30;
            for (int64_t sp = 1; sp <= std::min<int64_t>(P, std::max<int64_t>(1, nkb / 4)); ++sp) {
                const double cost = (double)ceil_div(tiles * sp, num_sms) * ((double)ceil_div(nkb, sp) + E);
                if (cost < best - 1e-9) { best = cost; sbest = sp; }
            }
            A.kb_per_split = (int)ceil_div(nkb, sbest);
            sbest = ceil_div(nkb, A.kb_per_split);
            A.cl = 0; A.zsplit = 0; A.atomic = 0; A.stg_bytes = 0;
            grid2((int)sbest);
            float* part = (float*)(ws + WL.b_off);
            A.out = part; A.alpha = 1.f; A.beta = 0.f; A.part_rows = g.k;  // slot = K x R*S*C (ldc = R*S*C)
            const int e = launch();
            if (e) return e;
            note_fused();
            return DRY(launch_partial_reduce((int)sbest, (int64_t)g.k * RSC, (int)RSC, g.k, (int)RSC, false, part,
                                             alpha, beta, (float*)out, st, mc_reduce));
        };
        if (algo == MUCU_ALGO_IM2COL_GEMM && i2c_implicit_wgrad(g)) {
            // I2C with the im2col done by the TMA unit (im2col mode) into shared memory, as
            // the implicit GEMM does; the workspace holds the split partials
            const int Pi = wgrad_implicit_slots(g);
            const bool part_ok = ctx->deterministic && Pi > 1;
            if (use_tma_im2col()) {
                wgrad_tiling(atom, true);
                if (!map_dy()) return -1;
                if (make_im2col_map(&L.tb, elt, in0, g.c, g.w, g.h, b, -g.pad, -g.pad, g.pad - (g.s - 1),
                                    g.pad - (g.r - 1), KB * A.km, g.stride, true)) {
                    A.tma_bytes = A.km * (A.mt * a_bytes + A.bn_atoms * KB * 128);
                    if (part_ok && A.cl)
                        return launch_partial(Pi, [&]() { return LAUNCH(A_TMA_MN2, B_TMA_IM2COL, EPI_WGRAD_PARTIAL); });
                    return LAUNCH(A_TMA_MN2, B_TMA_IM2COL, EPI_WGRAD_CHAIN);
                }
            }
            A.tma_bytes = a_bytes;
            wgrad_tiling(atom, false);
            if (!map_dy()) return -1;
            if (part_ok && A.cl)
                return launch_partial(Pi, [&]() { return LAUNCH(A_TMA_MN2, B_GATHER_WG, EPI_WGRAD_PARTIAL); });
            return LAUNCH(A_TMA_MN2, B_GATHER_WG, EPI_WGRAD_CHAIN);
        }
        if (algo == MUCU_ALGO_IM2COL_GEMM) {
            const void* colp = in0;
            int64_t kp = g.c;
            if (!is_pointwise(g)) {
                colp = ws + WL.a_off; kp = WL.kpitch;
                err = DRY(launch_im2col(g, b, in0, (void*)colp, (int)kp, st));
                if (err) return err;
            }
            if (RSC < atom) return -1;
            // dense (pointwise / explicit im2col) operands: single k-block stages keep a
            // deeper ring (deep ResNet 1x1 WGRAD -3..6 % against km = 2)
            wgrad_tiling(16, true, 0, env_int("MUCU_DENSE_KM", 1));
            if (!map_dy()) return -1;
            if (!map2(&L.tb, colp, RSC, (uint64_t)Mpix, kp, atom, KB * A.km, true)) return -1;
            map_mn_box(colp, RSC, (uint64_t)Mpix, kp, KB * A.km);
            A.tma_bytes = A.km * (A.mt * a_bytes + A.bn_atoms * KB * 128);
            if (ctx->deterministic && wgrad_partial_slots(g) > 1 && A.cl)
                return launch_partial(wgrad_partial_slots(g),
                                      [&]() { return LAUNCH(A_TMA_MN2, B_TMA_MN2, EPI_WGRAD_PARTIAL); });
            return LAUNCH(A_TMA_MN2, B_TMA_MN2, EPI_WGRAD_CHAIN);
        }
        // implicit-im2col B producers load whole 128-B channel atoms of one tap:
        // N tiles must start on an atom boundary.
        if (g.c % atom == 0 && use_tma_im2col()) {
            wgrad_tiling(atom, true);
            if (!map_dy()) return -1;
            if (make_im2col_map(&L.tb, elt, in0, g.c, g.w, g.h, b, -g.pad, -g.pad, g.pad - (g.s - 1),
                                g.pad - (g.r - 1), KB * A.km, g.stride, true)) {
                A.tma_bytes = A.km * (A.mt * a_bytes + A.bn_atoms * KB * 128);
                return LAUNCH(A_TMA_MN2, B_TMA_IM2COL, EPI_WGRAD_CHAIN);
            }
        }
        A.tma_bytes = a_bytes;
        if (g.c % atom == 0) {
            wgrad_tiling(atom, false);
            if (!map_dy()) return -1;
            return LAUNCH(A_TMA_MN2, B_GATHER_WG, EPI_WGRAD_CHAIN);
        }
        if (g.c * elt < 16) {
            // RGB-like layer: padded columns j' = (r, s8, c'), one 128-B atom per
            // 8-tap group; the epilogue folds them back into dw[k][r][s][c].
            A.cp = 16 / elt; A.s8 = (int)align_up((uint64_t)g.s, 8);
            A.N = g.r * A.s8 * A.cp;
            wgrad_tiling(atom, false);
            if (!map_dy()) return -1;
            return LAUNCH(A_TMA_MN2, B_GATHER_SMALLC, EPI_WGRAD_SMALLC);
        }
        wgrad_tiling(16, false);
        if (!map_dy()) return -1;
        return LAUNCH(A_TMA_MN2, B_SCALAR_WG, EPI_WGRAD_CHAIN);
    }
#undef LAUNCH
#undef DRY
    return -1;
}

}  // namespace mucu
