// api.cpp -- C ABI of libmucudnn (include/mucudnn.h): errors, geometry,
// workspace sizing, the handle, the micro-batch executor (Fig. 3),
// the benchmark pass (P:L88 WR step 1) and WD network planning
// (P:L163-167).
#include <cuda_runtime.h>
#include <cmath>

#include <algorithm>
#include <atomic>
#include <cstdarg>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <map>
#include <string>
#include <vector>

#include "mucudnn.h"
#include "mucudnn_internal.h"

namespace mucu {

static thread_local char g_err[512] = "";
static std::atomic<uint64_t> g_launches{0};

void count_launch() { g_launches.fetch_add(1, std::memory_order_relaxed); }

mucu_status_t set_error(mucu_status_t s, const char* fmt, ...) {
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(g_err, sizeof(g_err), fmt, ap);
    va_end(ap);
    return s;
}

static mucu_status_t cuda_error(int e, const char* where) {
    if (e == 0) return MUCU_OK;
    return set_error(MUCU_ERR_CUDA, "%s: %s", where, cudaGetErrorString((cudaError_t)e));
}

bool make_geom(const mucu_conv_desc_t* d, Geom* g) {
    if (!d) return false;
    if (d->n <= 0 || d->c <= 0 || d->h <= 0 || d->w <= 0 || d->k <= 0 || d->r <= 0 || d->s <= 0 ||
        d->pad < 0 || d->stride <= 0)
        return false;
    if (d->math < MUCU_MATH_F32 || d->math > MUCU_MATH_BF16) return false;
    g->n = d->n; g->c = d->c; g->h = d->h; g->w = d->w; g->k = d->k; g->r = d->r; g->s = d->s;
    g->pad = d->pad; g->stride = d->stride; g->math = d->math;
    int64_t pn = (int64_t)d->h + 2 * d->pad - d->r, qn = (int64_t)d->w + 2 * d->pad - d->s;
    if (pn < 0 || qn < 0) return false;
    g->p = (int32_t)(pn / d->stride + 1);
    g->q = (int32_t)(qn / d->stride + 1);
    return g->p > 0 && g->q > 0;
}

bool is_pointwise(const Geom& g) { return g.r == 1 && g.s == 1 && g.pad == 0 && g.stride == 1; }

bool small_c_tc(const Geom& g) { return g.math != MUCU_MATH_F32 && g.c * elt_size(g.math) < 16; }

bool i2c_implicit_wgrad(const Geom& g) {
    return g.math != MUCU_MATH_F32 && !is_pointwise(g) && g.c % (128 / elt_size(g.math)) == 0;
}

int wgrad_implicit_slots(const Geom& g) {
    const int64_t tiles = ceil_div(g.k, 256) * ceil_div((int64_t)g.r * g.s * g.c, 256);
    return (int)std::max<int64_t>(1, std::min<int64_t>(kPartialSlots, ceil_div(kPartialSlots, tiles)));
}

int s2d_channels(const Geom& g) {
    const int atom = 128 / elt_size(g.math);
    return (int)align_up((uint64_t)g.stride * g.stride * g.c, (uint64_t)atom);
}

S2d s2d_geom(const Geom& g, int type) {
    S2d z;
    const int st = g.stride;
    const int atom = 128 / elt_size(g.math);
    if (type == MUCU_BWD_DATA) {
        // dx super-pixels of f = st*u rows/cols; dx row f*i + a' - pad takes dy rows
        // p = u*i + u-1-d (d < Dr = ceil(R/st) - 1 + u) through filter row
        // r = st*d + a' - st*(u-1).  u = 2 when f*f*C stays <= 256 GEMM columns.
        z.u = 2;
        while (z.u > 1 && st * z.u * st * z.u * g.c > 256) --z.u;
        z.f = st * z.u;
        z.Dr = (g.r - 1) / st + z.u;
        z.Ds = (g.s - 1) / st + z.u;
        z.Cs = 0;
        z.I = (g.h - 1 + g.pad) / z.f + 1;
        z.J = (g.w - 1 + g.pad) / z.f + 1;
        z.Pu = z.Qu = 0;
        return z;
    }
    // FWD / WGRAD: output super-pixels of u x u (u = 2 for FWD: N = 4K columns)
    z.u = type == MUCU_FWD ? 2 : 1;
    z.f = st * z.u;
    // output row u*i' + uu reads input rows f*(i' + d) + a - pad with st*uu + r = f*d + a
    z.Dr = (st * (z.u - 1) + g.r - 1) / z.f + 1;
    z.Ds = (st * (z.u - 1) + g.s - 1) / z.f + 1;
    z.Cs = (int)align_up((uint64_t)z.f * z.f * g.c, (uint64_t)atom);
    z.Pu = (g.p + z.u - 1) / z.u;
    z.Qu = (g.q + z.u - 1) / z.u;
    z.I = z.Pu + z.Dr - 1;
    z.J = z.Qu + z.Ds - 1;
    return z;
}

bool s2d_tc(const Geom& g, int type) {
    if (!small_c_tc(g) || g.stride < 2) return false;
    if (type == MUCU_BWD_DATA) return g.k % (128 / elt_size(g.math)) == 0 && g.stride * g.stride * g.c <= 256;
    // (DGRAD: s2d_geom picks the largest u <= 2 with (st*u)^2 * C <= 256 columns)
    // even 12 -> 64 padded channels (ResNet conv1, BF16) run ~5-8x faster on
    // the TMA-fed space-to-depth GEMM than on the 16-B tap gathers
    return true;
}

bool win_tc(const Geom& g, int type) {
    const int elt = elt_size(g.math);
    return type == MUCU_BWD_FILTER && small_c_tc(g) && g.stride >= 2 && g.c <= 4 &&
           (g.stride * 4 * elt) % 16 == 0;
}

int wgrad_partial_slots(const Geom& g) {
    if (g.math == MUCU_MATH_F32) return 1;
    const int64_t tiles = ceil_div(g.k, 128) * ceil_div((int64_t)g.r * g.s * g.c, 128);
    return (int)std::max<int64_t>(1, std::min<int64_t>(kPartialSlots, ceil_div(kPartialSlots, tiles)));
}

bool staged_wg_geom(const Geom& g, StagedWg* z) {
    if (!small_c_tc(g)) return false;
    const int elt = elt_size(g.math), KB = 128 / elt, atom = 128 / elt;
    const int64_t RSC = (int64_t)g.r * g.s * g.c;
    z->TR = (int)align_up((uint64_t)RSC, 128);
    z->mt = z->TR / 128;
    z->kd = KB;
    const int WC = g.w * g.c;
    const int span = (g.stride * (KB - 1) + g.s) * g.c;  // elements a pixel block reads per x row
    z->cs = 0; z->bch = 0;
    for (int c = 256; c >= 1; --c) {
        if (WC % c || (c * elt) % 16) continue;
        const int bc = (span + 2 * (c - 1)) / c;  // any start offset inside a chunk
        if (!z->cs || (int64_t)bc * c < (int64_t)z->bch * z->cs) { z->cs = c; z->bch = bc; }
    }
    z->b_bytes = std::max(g.k * 128, (g.k * elt / 128) * KB * 128);
    z->sx_tx = g.r * z->bch * z->cs * elt;
    z->sx_bytes = (int)align_up((uint64_t)z->sx_tx, 1024);
    z->tab_bytes = (int)align_up((uint64_t)z->TR * 4, 1024);
    const int stage = z->mt * 16384 + z->b_bytes;
    z->Ss = 0; z->SX = 0;
    for (int sa : {2, 3})
        for (int sx : {8, 6, 5, 4, 3, 2})
            if (!z->Ss && sa * stage + sx * z->sx_bytes + z->tab_bytes <= 210 * 1024) { z->Ss = sa; z->SX = sx; }
    // taps padded to whole 128-row halves: more than a quarter of padding rows (ResNet 7x7x3:
    // 147 -> 256) costs more MMA and builder time than the window form saves (measured:
    // ResNet-18/50 conv1 BF16 0.47 ms staged vs 0.32 ms window; AlexNet 363 -> 384 gains)
    return z->mt <= 4 && g.k <= 256 && g.k % atom == 0 && z->cs > 0 && g.r <= 256 && z->bch <= 256 && z->Ss &&
           128 * z->mt * (g.k + 4) * 4 <= 210 * 1024 && (z->TR - RSC) * 4 <= RSC;
}

Win win_geom(const Geom& g) {
    Win z;
    const int elt = elt_size(g.math);
    z.cpx = 4;
    // GEMM rows per filter row = na * aw/elt; BF16 may use 64- or 32-B swizzle atoms
    // (fewer padded taps: ResNet 7 taps -> one 8-tap 64-B atom instead of a 16-tap
    // 128-B one); TF32 MN-major operands need the 128-B (32-B-base) layout.
    z.aw = 128;
    int best = 1 << 30;
    for (int aw = 128; aw >= (elt == 2 ? 32 : 128); aw /= 2) {
        const int tpa = aw / elt / z.cpx, na = (g.s + tpa - 1) / tpa;
        const int M = (int)align_up((uint64_t)g.r * na * (aw / elt), 256);
        if (M < best) { best = M; z.aw = aw; }
    }
    z.tpa = z.aw / elt / z.cpx;
    z.na = (g.s + z.tpa - 1) / z.tpa;
    // every window read stays inside its row: st*(Q-1) + na*tpa <= Wp
    z.Wp = (int)align_up((uint64_t)std::max(g.stride * (g.q - 1) + z.na * z.tpa, g.w + g.pad), 4);
    z.M = g.r * z.na * (z.aw / elt);
    return z;
}

bool algo_eligible(const Geom& g, int type, int algo) {
    if (type < MUCU_FWD || type > MUCU_BWD_FILTER) return false;
    switch (algo) {
        case MUCU_ALGO_IMPLICIT_GEMM:
        case MUCU_ALGO_IM2COL_GEMM:
            return true;
        case MUCU_ALGO_WINOGRAD_2X2_3X3:
            // F(2x2,3x3): 3x3 filters, unit stride (ref [23]); pad' = 2 - pad >= 0 for
            // DGRAD.  BackwardFilter runs the transposed F(3x3,2x2).
            return g.r == 3 && g.s == 3 && g.stride == 1 && g.pad <= 2;
        case MUCU_ALGO_FFT:
        case MUCU_ALGO_FFT_TILING: {
            FftGeom z;
            return fft_geom(g, type, algo, &z);
        }
        default:
            return false;
    }
}

mucu_status_t ws_layout(const Geom& g, int type, int algo, int32_t b, WsLayout* L) {
    std::memset(L, 0, sizeof(*L));
    if (!algo_eligible(g, type, algo)) return set_error(MUCU_ERR_UNSUPPORTED, "algorithm %d ineligible for this layer/type", algo);
    if (b <= 0 || b > g.n) return set_error(MUCU_ERR_INVALID_VALUE, "micro-batch size %d outside 1..%d", b, g.n);
    const uint64_t elt = (uint64_t)elt_size(g.math);
    const uint64_t vec = 16 / elt;
    const uint64_t RSC = (uint64_t)g.r * g.s * g.c;
    const uint64_t PQ = (uint64_t)g.p * g.q;
    if (algo == MUCU_ALGO_IMPLICIT_GEMM) return MUCU_OK;
    if (algo == MUCU_ALGO_IM2COL_GEMM) {
        L->kpitch = (int32_t)align_up(RSC, vec);
        // tensor-core BackwardFilter: partial dW slots [P][K][R*S*C] fp32 after the col buffer
        const int P = type == MUCU_BWD_FILTER ? wgrad_partial_slots(g) : 1;
        const uint64_t part = P > 1 ? align_up((uint64_t)P * g.k * RSC * 4, 256) : 0;
        if (is_pointwise(g)) {
            L->kpitch = g.c;
            L->b_off = 0; L->b_bytes = part; L->total = part;
            return MUCU_OK;
        }
        if (type == MUCU_BWD_FILTER && i2c_implicit_wgrad(g)) {
            // TMA im2col into shared memory: only the per-split partial dW slots
            const int Pi = wgrad_implicit_slots(g);
            L->a_off = 0; L->a_bytes = 0;
            L->b_off = 0; L->b_bytes = Pi > 1 ? align_up((uint64_t)Pi * g.k * RSC * 4, 256) : 0;
            L->total = L->b_bytes;
            return MUCU_OK;
        }
        StagedWg sw;
        if (type == MUCU_BWD_FILTER && staged_wg_geom(g, &sw)) {
            // staged-row kernel + per-split partial dW tiles (b-independent)
            L->a_off = 0;
            L->a_bytes = align_up((uint64_t)kPartialSlots * sw.TR * g.k * 4, 256);
            L->kpitch = 0;
            L->total = L->a_bytes;
            return MUCU_OK;
        }
        if (win_tc(g, type)) {
            // padded x, then (deterministic split-K) kPartialSlots partial dW tiles of
            // z.M window rows x K filters fp32 (b-independent)
            const Win z = win_geom(g);
            L->a_off = 0;
            L->a_bytes = align_up((uint64_t)b * g.h * z.Wp * z.cpx * elt, 256);
            L->b_off = L->a_bytes;
            L->b_bytes = align_up((uint64_t)kPartialSlots * z.M * g.k * 4, 256);
            L->kpitch = z.cpx;
            L->total = L->a_bytes + L->b_bytes;
            return MUCU_OK;
        }
        if (s2d_tc(g, type)) {
            // Space-to-depth: FWD = [s2d filter K x Dr*Ds*Cs][xs b x I x J x Cs],
            // WGRAD = [xs], DGRAD = [s2d filter st*st*C x Dr*Ds*K] (b-independent).
            const S2d z = s2d_geom(g, type);
            const uint64_t Dr = z.Dr, Ds = z.Ds, Cs = z.Cs;
            if (type == MUCU_BWD_DATA) {
                L->fixed_bytes = align_up((uint64_t)z.f * z.f * g.c * Dr * Ds * g.k * elt, 256);
            } else {
                if (type == MUCU_FWD)
                    L->fixed_bytes = align_up((uint64_t)z.u * z.u * g.k * Dr * Ds * Cs * elt, 256);
                L->a_off = L->fixed_bytes;
                L->a_bytes = align_up((uint64_t)b * z.I * z.J * Cs * elt, 256);
            }
            L->kpitch = (int32_t)Cs;
            L->total = L->fixed_bytes + L->a_bytes;
            return MUCU_OK;
        }
        if (small_c_tc(g) && type != MUCU_BWD_DATA) {
            // Tensor-core small-C (RGB) layers: the explicit transform is a
            // channel pad of x to 16 B per pixel (the GEMM walks the taps);
            // b*H*W*16 bytes instead of the full b*P*Q*R*S*C im2col matrix.
            L->kpitch = 16 / (int32_t)elt;
            L->a_off = 0;
            L->a_bytes = align_up((uint64_t)b * g.h * g.w * 16, 256);
            L->total = L->a_bytes;
            return MUCU_OK;
        }
        if (type == MUCU_BWD_DATA) {
            // tensor cores read the filter as MN-major 128-B atoms: rows shorter
            // than one atom are padded to it
            const bool short_row = g.math != MUCU_MATH_F32 && RSC < 128 / elt;
            L->filter_padded = (RSC * elt) % 16 != 0 || short_row;
            const uint64_t fpitch = short_row ? 128 / elt : align_up(RSC, vec);
            L->fixed_bytes = L->filter_padded ? align_up((uint64_t)g.k * fpitch * elt, 256) : 0;
            L->kpitch = (int32_t)align_up(RSC, 4);  // fp32 dcol
            L->a_off = L->fixed_bytes;
            L->a_bytes = align_up((uint64_t)b * PQ * (uint64_t)L->kpitch * 4, 256);
        } else {
            L->filter_padded = (type == MUCU_FWD) && (RSC * elt) % 16 != 0;
            L->fixed_bytes = L->filter_padded ? align_up((uint64_t)g.k * L->kpitch * elt, 256) : 0;
            L->a_off = L->fixed_bytes;
            L->a_bytes = align_up((uint64_t)b * PQ * (uint64_t)L->kpitch * elt, 256);
        }
        L->b_off = L->a_off + L->a_bytes;
        L->b_bytes = part;
        L->total = L->b_off + L->b_bytes;
        return MUCU_OK;
    }
    if (algo == MUCU_ALGO_FFT || algo == MUCU_ALGO_FFT_TILING) {
        // spectra (complex fp32): filter [bins][K][C] | input tiles | output tiles
        // (WGRAD: dW spectrum | x tiles | dy tiles -- the spectrum first, at an offset
        // independent of b, so consecutive micro-batches accumulate into it).  DESIGN.md 6.11.
        FftGeom z;
        fft_geom(g, type, algo, &z);
        const uint64_t B = (uint64_t)z.bins, Pl = (uint64_t)b * z.tiles_y * z.tiles_x;
        const uint64_t KC = align_up(8 * B * g.k * g.c, 256);
        const uint64_t in_ch = type == MUCU_FWD ? g.c : (uint64_t)g.k;   // x (FWD, WGRAD a) / dy (DGRAD)
        const uint64_t out_ch = type == MUCU_FWD ? g.k : (uint64_t)g.c;
        if (type == MUCU_BWD_FILTER) {
            L->fixed_off = 0;  // dW spectrum (accumulated over a run of micro-batches)
            L->fixed_bytes = KC;
            L->a_off = KC;
            L->a_bytes = align_up(8 * B * Pl * g.c, 256);
            L->b_off = L->a_off + L->a_bytes;
            L->b_bytes = align_up(8 * B * Pl * g.k, 256);
            L->total = L->b_off + L->b_bytes;
            return MUCU_OK;
        }
        L->fixed_off = 0;
        L->fixed_bytes = KC;
        L->a_off = KC;
        L->a_bytes = align_up(8 * B * Pl * in_ch, 256);
        L->b_off = L->a_off + L->a_bytes;
        L->b_bytes = align_up(8 * B * Pl * out_ch, 256);
        L->total = L->b_off + L->b_bytes;
        return MUCU_OK;
    }
    if (type == MUCU_BWD_FILTER) {
        // Winograd F(3x3,2x2) BackwardFilter: V = B^T x B [16][Tp][C] | D = A dy A^T
        // [16][Tp][K] | M [16][K][C] fp32; T = b*ceil(P/2)*ceil(Q/2) tiles padded to
        // Tp = a multiple of 256 (zero rows: whole TMA k-blocks per plane).
        // Channel pitches Cp, Kp: C, K rounded up to 128 B (zero channels), the TMA atom.
        const uint64_t Tp = align_up((uint64_t)b * ((g.p + 1) / 2) * ((g.q + 1) / 2), 256);
        const uint64_t Cp = align_up((uint64_t)g.c, 128 / elt), Kp = align_up((uint64_t)g.k, 128 / elt);
        L->a_off = 0;
        L->a_bytes = align_up(16 * Tp * Cp * elt, 256);
        L->b_off = L->a_bytes;
        L->b_bytes = align_up(16 * Tp * Kp * elt, 256);
        L->fixed_off = L->b_off + L->b_bytes;  // M (per call, not b-independent)
        L->total = L->fixed_off + align_up(16 * Kp * Cp * 4, 256);
        return MUCU_OK;
    }
    // Winograd F(2x2,3x3): U (b-independent) | V | M (fp32).
    const bool dgrad = type == MUCU_BWD_DATA;
    const uint64_t OH = dgrad ? g.h : g.p, OW = dgrad ? g.w : g.q;
    const uint64_t I = dgrad ? g.k : g.c, O = dgrad ? g.c : g.k;
    const uint64_t T = ((OH + 1) / 2) * ((OW + 1) / 2);
    L->fixed_bytes = align_up(16 * O * I * elt, 256);
    L->a_off = L->fixed_bytes;
    L->a_bytes = align_up(16 * (uint64_t)b * T * I * elt, 256);
    L->b_off = L->a_off + L->a_bytes;
    L->b_bytes = align_up(16 * (uint64_t)b * T * O * 4, 256);
    L->total = L->b_off + L->b_bytes;
    return MUCU_OK;
}

struct Handle {
    int device = 0;
    int num_sms = 148;
    int policy = MUCU_POLICY_POW2;
    int warmup = 2, reps = 5;
    bool deterministic = true;  // BackwardFilter split-K order (mucu_set_deterministic)
    std::map<std::string, std::pair<std::vector<int64_t>, std::vector<uint64_t>>> cache;
    // (descriptor, type, algo, b) -> tensor-core path available (executor pre-validation)
    std::map<std::string, bool> tc_ok;
};

static bool tc_math(int math) { return math == MUCU_MATH_TF32 || math == MUCU_MATH_BF16; }

// ------------------------------------------------------------- dispatch --
mucu_status_t run_micro(Handle* hd, const Geom& g, int type, int algo, int32_t b, float alpha, const void* in0,
                        const void* in1, float beta, void* out, void* ws, uint64_t ws_bytes, cudaStream_t st,
                        CallCtx* ctx) {
    WsLayout L;
    mucu_status_t s = ws_layout(g, type, algo, b, &L);
    if (s != MUCU_OK) return s;
    if (L.total > ws_bytes) return set_error(MUCU_ERR_INSUFFICIENT_WORKSPACE, "workspace %llu < %llu", (unsigned long long)ws_bytes, (unsigned long long)L.total);
    char* wsb = (char*)ws;
    const bool tc = tc_math(g.math);
    // The b-independent workspace prefix (padded filter / Winograd U / space-to-depth
    // filter) computed by an earlier micro-config of this call stays valid only while
    // the same algorithm runs: any other algorithm may write its own segments over it.
    if (ctx->last_algo != algo) {
        ctx->fixed_kind = 0;
        ctx->fixed_src = nullptr;
        ctx->last_algo = algo;
    }
    ctx->deterministic = hd->deterministic;
    int e = 0;
    if (tc) {
        e = tc_run_micro(g, type, algo, b, alpha, in0, in1, beta, out, wsb, L, hd->num_sms, st, ctx);
        if (e == -1) return set_error(MUCU_ERR_UNSUPPORTED, "tensor-core path not available for this configuration");
        return cuda_error(e, "tc kernel");
    }
    // ---- MUCU_MATH_F32: SIMT FFMA ----
    const float* f0 = (const float*)in0;
    const float* f1 = (const float*)in1;
    float* fo = (float*)out;
    if (algo == MUCU_ALGO_FFT || algo == MUCU_ALGO_FFT_TILING) {
        if (ctx->dry) return MUCU_OK;
        e = fft_run(g, type, algo, b, alpha, f0, f1, beta, fo, wsb, L, ctx, st);
        if (e == -1) return set_error(MUCU_ERR_UNSUPPORTED, "FFT path not available for this configuration");
        return cuda_error(e, "fft kernel");
    }
    if (type == MUCU_FWD) {
        if (algo == MUCU_ALGO_IMPLICIT_GEMM) {
            e = simt_fwd_ig(g, b, alpha, f0, f1, beta, fo, st);
        } else if (algo == MUCU_ALGO_IM2COL_GEMM) {
            const int64_t M = (int64_t)b * g.p * g.q, Kd = (int64_t)g.r * g.s * g.c;
            if (is_pointwise(g)) {
                e = simt_gemm_nt(M, g.k, Kd, alpha, f0, g.c, f1, Kd, beta, fo, g.k, 1, 0, 0, 0, st);
            } else {
                float* col = (float*)(wsb + L.a_off);
                e = launch_im2col(g, b, f0, col, L.kpitch, st);
                if (!e) e = simt_gemm_nt(M, g.k, Kd, alpha, col, L.kpitch, f1, Kd, beta, fo, g.k, 1, 0, 0, 0, st);
            }
        } else {
            e = 0;
            if (ctx->fixed_kind != 2 || ctx->fixed_src != in1) {
                e = launch_wg_filter(g, false, f1, wsb, st);
                ctx->fixed_kind = 2; ctx->fixed_src = in1;
            }
            const int64_t T = (int64_t)((g.p + 1) / 2) * ((g.q + 1) / 2) * b;
            float* V = (float*)(wsb + L.a_off);
            float* Mx = (float*)(wsb + L.b_off);
            if (!e) e = launch_wg_input(g, false, b, f0, V, st);
            if (!e) e = simt_gemm_nt(T, g.k, g.c, 1.f, V, g.c, (const float*)wsb, g.c, 0.f, Mx, g.k, 16,
                                     T * g.c, (int64_t)g.k * g.c, T * g.k, st);
            if (!e) e = launch_wg_output(g, false, b, alpha, Mx, beta, fo, st);
        }
    } else if (type == MUCU_BWD_DATA) {
        if (algo == MUCU_ALGO_IMPLICIT_GEMM) {
            e = (g.c <= 4 && !(getenv("MUCU_SMALLC_DGRAD") && atoi(getenv("MUCU_SMALLC_DGRAD")) == 0))
                    ? small_c_dgrad(g, b, alpha, f0, f1, beta, fo, st) : -1;
            if (e == -1) e = simt_dgrad_ig(g, b, alpha, f0, f1, beta, fo, st);
        } else if (algo == MUCU_ALGO_IM2COL_GEMM) {
            const int64_t M = (int64_t)b * g.p * g.q, RSC = (int64_t)g.r * g.s * g.c;
            if (is_pointwise(g)) {
                e = simt_gemm_nn(M, g.c, g.k, alpha, f0, g.k, f1, g.c, beta, fo, g.c, st);
            } else {
                float* dcol = (float*)(wsb + L.a_off);
                e = simt_gemm_nn(M, RSC, g.k, 1.f, f0, g.k, f1, RSC, 0.f, dcol, L.kpitch, st);
                if (!e) e = launch_col2im(g, b, alpha, dcol, L.kpitch, beta, fo, st);
            }
        } else {
            if (ctx->fixed_kind != 2 || ctx->fixed_src != in1) {
                e = launch_wg_filter(g, true, f1, wsb, st);
                ctx->fixed_kind = 2; ctx->fixed_src = in1;
            }
            const int64_t T = (int64_t)((g.h + 1) / 2) * ((g.w + 1) / 2) * b;
            float* V = (float*)(wsb + L.a_off);
            float* Mx = (float*)(wsb + L.b_off);
            if (!e) e = launch_wg_input(g, true, b, f0, V, st);
            if (!e) e = simt_gemm_nt(T, g.c, g.k, 1.f, V, g.k, (const float*)wsb, g.k, 0.f, Mx, g.c, 16,
                                     T * g.k, (int64_t)g.c * g.k, T * g.c, st);
            if (!e) e = launch_wg_output(g, true, b, alpha, Mx, beta, fo, st);
        }
    } else {  // MUCU_BWD_FILTER: in0 = x, in1 = dy, out = dw (fp32)
        if (algo == MUCU_ALGO_WINOGRAD_2X2_3X3) {
            // M_xi[k][c] = sum_t D[xi][t][k] V[xi][t][c] (16 batched GEMMs over the tiles)
            const int64_t Tp = (int64_t)align_up((uint64_t)b * ((g.p + 1) / 2) * ((g.q + 1) / 2), 256);
            float* V = (float*)(wsb + L.a_off);
            float* D = (float*)(wsb + L.b_off);
            float* Mx = (float*)(wsb + L.fixed_off);
            e = launch_wgw_transforms(g, b, f0, f1, V, D, Tp, st);
            if (!e) e = simt_gemm_tt(g.k, g.c, Tp, V, D, Mx, Tp, st);  // F32: Cp = C, Kp = K (mult. of 32 or padded)
            if (!e) e = launch_wgw_output(g, alpha, Mx, beta, fo, st);
        } else if (algo == MUCU_ALGO_IMPLICIT_GEMM) {
            e = simt_wgrad(g, b, alpha, f1, f0, false, 0, beta, fo, hd->num_sms, st);
        } else {
            if (is_pointwise(g)) {
                e = simt_wgrad(g, b, alpha, f1, f0, true, g.c, beta, fo, hd->num_sms, st);
            } else {
                float* col = (float*)(wsb + L.a_off);
                e = launch_im2col(g, b, f0, col, L.kpitch, st);
                if (!e) e = simt_wgrad(g, b, alpha, f1, col, true, L.kpitch, beta, fo, hd->num_sms, st);
            }
        }
    }
    return cuda_error(e, "simt kernel");
}

}  // namespace mucu

using namespace mucu;

struct mucu_handle : public mucu::Handle {};

struct mucu_network {
    struct Kernel {
        mucu_conv_desc_t desc;
        int type;
        std::vector<mucu_micro_config_t> plan;
        uint64_t offset = 0, bytes = 0;
        int64_t time_ns = 0;
    };
    std::vector<Kernel> kernels;
    bool planned = false;
};

// ================================================================= misc ====
extern "C" const char* mucu_status_string(mucu_status_t s) {
    switch (s) {
        case MUCU_OK: return "MUCU_OK";
        case MUCU_ERR_INVALID_VALUE: return "MUCU_ERR_INVALID_VALUE";
        case MUCU_ERR_UNSUPPORTED: return "MUCU_ERR_UNSUPPORTED";
        case MUCU_ERR_INSUFFICIENT_WORKSPACE: return "MUCU_ERR_INSUFFICIENT_WORKSPACE";
        case MUCU_ERR_INFEASIBLE: return "MUCU_ERR_INFEASIBLE";
        case MUCU_ERR_CAPACITY: return "MUCU_ERR_CAPACITY";
        case MUCU_ERR_MISALIGNED: return "MUCU_ERR_MISALIGNED";
        case MUCU_ERR_CUDA: return "MUCU_ERR_CUDA";
        case MUCU_ERR_INTERNAL: return "MUCU_ERR_INTERNAL";
    }
    return "MUCU_ERR_UNKNOWN";
}

extern "C" const char* mucu_last_error(mucu_handle_t) { return g_err; }
extern "C" int32_t mucu_version(void) { return MUCU_VERSION; }
extern "C" uint64_t mucu_launch_count(void) { return g_launches.load(std::memory_order_relaxed); }

static int policy_from_env(int dflt) {
    const char* p = getenv("MUCU_BATCH_POLICY");
    if (!p) return dflt;
    if (!strcmp(p, "all")) return MUCU_POLICY_ALL;
    if (!strcmp(p, "pow2") || !strcmp(p, "powerOfTwo")) return MUCU_POLICY_POW2;
    if (!strcmp(p, "undivided")) return MUCU_POLICY_UNDIVIDED;
    return dflt;
}

extern "C" mucu_status_t mucu_create(mucu_handle_t* out, int device) {
    if (!out) return set_error(MUCU_ERR_INVALID_VALUE, "create: null handle pointer");
    *out = nullptr;
    int e = (int)cudaSetDevice(device);
    if (e) return cuda_error(e, "cudaSetDevice");
    mucu_handle* h = new (std::nothrow) mucu_handle();
    if (!h) return set_error(MUCU_ERR_INTERNAL, "create: out of host memory");
    h->device = device;
    cudaDeviceGetAttribute(&h->num_sms, cudaDevAttrMultiProcessorCount, device);
    h->policy = policy_from_env(MUCU_POLICY_POW2);
    if (const char* w = getenv("MUCU_BENCH_WARMUP")) h->warmup = std::max(0, atoi(w));
    if (const char* r = getenv("MUCU_BENCH_REPS")) h->reps = std::max(1, atoi(r));
    if (const char* dt = getenv("MUCU_DETERMINISTIC")) h->deterministic = atoi(dt) != 0;
    *out = h;
    return MUCU_OK;
}

extern "C" mucu_status_t mucu_destroy(mucu_handle_t h) {
    if (!h) return MUCU_OK;
    delete h;
    return MUCU_OK;
}

extern "C" mucu_status_t mucu_set_policy(mucu_handle_t h, mucu_policy_t p) {
    if (!h || p < MUCU_POLICY_ALL || p > MUCU_POLICY_UNDIVIDED) return set_error(MUCU_ERR_INVALID_VALUE, "set_policy");
    h->policy = p;
    return MUCU_OK;
}

extern "C" mucu_status_t mucu_set_deterministic(mucu_handle_t h, int32_t deterministic) {
    if (!h) return set_error(MUCU_ERR_INVALID_VALUE, "set_deterministic: null handle");
    h->deterministic = deterministic != 0;
    h->tc_ok.clear();
    return MUCU_OK;
}

extern "C" mucu_status_t mucu_set_bench_params(mucu_handle_t h, int32_t warmup, int32_t reps) {
    if (!h || warmup < 0 || reps < 1) return set_error(MUCU_ERR_INVALID_VALUE, "set_bench_params");
    h->warmup = warmup;
    h->reps = reps;
    return MUCU_OK;
}

extern "C" mucu_status_t mucu_output_dims(const mucu_conv_desc_t* d, int32_t* p, int32_t* q) {
    Geom g;
    if (!make_geom(d, &g) || !p || !q) return set_error(MUCU_ERR_INVALID_VALUE, "output_dims: invalid descriptor");
    *p = g.p;
    *q = g.q;
    return MUCU_OK;
}

extern "C" mucu_status_t mucu_workspace_size(const mucu_conv_desc_t* d, mucu_conv_type_t type, mucu_algo_t algo,
                                             int32_t micro_n, uint64_t* bytes) {
    Geom g;
    if (!make_geom(d, &g) || !bytes) return set_error(MUCU_ERR_INVALID_VALUE, "workspace_size: invalid descriptor");
    WsLayout L;
    mucu_status_t s = ws_layout(g, type, algo, micro_n, &L);
    if (s == MUCU_OK) *bytes = L.total;
    return s;
}

// ============================================================= executor ====
static mucu_status_t check_ptr(const void* p, const char* what) {
    if (!p) return set_error(MUCU_ERR_INVALID_VALUE, "%s is null", what);
    if ((uintptr_t)p % 16) return set_error(MUCU_ERR_MISALIGNED, "%s not 16-byte aligned", what);
    return MUCU_OK;
}

static mucu_status_t execute(mucu_handle_t h, const mucu_conv_desc_t* d, int type, const mucu_micro_config_t* plan,
                             int32_t count, float alpha, const void* in0, const void* in1, float beta, void* out,
                             void* ws, uint64_t ws_bytes, void* stream, const RedTarget* red = nullptr) {
    if (!h) return set_error(MUCU_ERR_INVALID_VALUE, "null handle");
    Geom g;
    if (!make_geom(d, &g)) return set_error(MUCU_ERR_INVALID_VALUE, "invalid descriptor");
    if (!plan || count <= 0) return set_error(MUCU_ERR_INVALID_VALUE, "empty plan");
    mucu_status_t s;
    if ((s = check_ptr(in0, "input 0")) || (s = check_ptr(in1, "input 1")) || (s = check_ptr(out, "output"))) return s;
    if (ws && (uintptr_t)ws % 256) return set_error(MUCU_ERR_MISALIGNED, "workspace not 256-byte aligned");
    // Validate the whole plan before any launch.
    int64_t sum = 0;
    for (int32_t i = 0; i < count; ++i) {
        if (plan[i].micro_n <= 0) return set_error(MUCU_ERR_INVALID_VALUE, "plan part %d has micro_n <= 0", i);
        sum += plan[i].micro_n;
        if (sum > g.n) return set_error(MUCU_ERR_INVALID_VALUE, "plan parts exceed N");
        WsLayout L;
        if ((s = ws_layout(g, type, plan[i].algo, plan[i].micro_n, &L))) return s;
        if (L.total > ws_bytes || (L.total && !ws))
            return set_error(MUCU_ERR_INSUFFICIENT_WORKSPACE, "part %d needs %llu workspace bytes, have %llu", i,
                             (unsigned long long)L.total, (unsigned long long)ws_bytes);
    }
    if (sum != g.n) return set_error(MUCU_ERR_INVALID_VALUE, "plan parts sum to %lld, N = %d", (long long)sum, g.n);
    const uint64_t elt = (uint64_t)elt_size(g.math);
    const uint64_t in_sample = (uint64_t)g.h * g.w * g.c * elt;   // x / dx per sample
    const uint64_t out_sample = (uint64_t)g.p * g.q * g.k * elt;  // y / dy per sample
    cudaStream_t st = (cudaStream_t)stream;
    auto part_ptrs = [&](int32_t i, int64_t done, const char*& p0, const char*& p1, char*& po, float& bta) {
        p0 = (const char*)in0; p1 = (const char*)in1; po = (char*)out; bta = beta;
        if (type == MUCU_FWD) { p0 += done * in_sample; po += done * out_sample; }
        else if (type == MUCU_BWD_DATA) { p0 += done * out_sample; po += done * in_sample; }
        else { p0 += done * in_sample; p1 += done * out_sample; if (i > 0) bta = 1.f; }  // P:L58 output scale
    };
    // Tensor-core eligibility of every part before the first launch (a dry run of
    // the dispatch: tilings, shared-memory budget, tensor-map encodings), cached per
    // (descriptor, type, algorithm, b) -- a failure mid-plan would leave y / dx / dw
    // partially updated.
    if (tc_math(g.math)) {
        int64_t done = 0;
        for (int32_t i = 0; i < count; ++i) {
            char key[160];
            snprintf(key, sizeof(key), "%d,%d,%d,%d,%d,%d,%d,%d,%d,%d|%d|%d|%d", d->n, d->c, d->h, d->w, d->k, d->r,
                     d->s, d->pad, d->stride, d->math, type, plan[i].algo, plan[i].micro_n);
            auto it = h->tc_ok.find(key);
            bool ok;
            if (it != h->tc_ok.end()) {
                ok = it->second;
            } else {
                const char *p0, *p1;
                char* po;
                float bta;
                part_ptrs(i, done, p0, p1, po, bta);
                CallCtx dry;
                dry.dry = true;
                ok = run_micro(h, g, type, plan[i].algo, plan[i].micro_n, alpha, p0, p1, bta, po, ws, ws_bytes, st,
                               &dry) == MUCU_OK;
                h->tc_ok[key] = ok;
            }
            if (!ok)
                return set_error(MUCU_ERR_UNSUPPORTED, "plan part %d (algo %d, b = %d): no tensor-core kernel for this "
                                 "configuration", i, plan[i].algo, plan[i].micro_n);
            done += plan[i].micro_n;
        }
    }
    CallCtx ctx;
    if (red) ctx.red = *red;
    int64_t done = 0;
    for (int32_t i = 0; i < count; ++i) {
        const int32_t b = plan[i].micro_n;
        const char *p0, *p1;
        char* po;
        float bta;
        part_ptrs(i, done, p0, p1, po, bta);
        ctx.mc_last = i == count - 1;
        ctx.next_algo = i + 1 < count ? plan[i + 1].algo : -1;
        s = run_micro(h, g, type, plan[i].algo, b, alpha, p0, p1, bta, po, ws, ws_bytes, st, &ctx);
        if (s) return s;
        done += b;
    }
    if (red && !ctx.mc_fused) {
        // NEXT-3: the last micro-configuration's dw writer did not take the reduction
        // (F32 SIMT, Winograd, FFT, atomic split-K): push the final dw
        const int e = launch_reduce_push((const float*)out, *red, (int64_t)g.k * g.r * g.s * g.c, st);
        if (e) return set_error(MUCU_ERR_CUDA, "reduce push: %s", cudaGetErrorString((cudaError_t)e));
    }
    return MUCU_OK;
}

extern "C" mucu_status_t mucu_conv_forward(mucu_handle_t h, const mucu_conv_desc_t* d, const mucu_micro_config_t* plan,
                                           int32_t count, float alpha, const void* x, const void* w, float beta,
                                           void* y, void* ws, uint64_t ws_bytes, void* stream) {
    return execute(h, d, MUCU_FWD, plan, count, alpha, x, w, beta, y, ws, ws_bytes, stream);
}

extern "C" mucu_status_t mucu_conv_backward_data(mucu_handle_t h, const mucu_conv_desc_t* d,
                                                 const mucu_micro_config_t* plan, int32_t count, float alpha,
                                                 const void* dy, const void* w, float beta, void* dx, void* ws,
                                                 uint64_t ws_bytes, void* stream) {
    return execute(h, d, MUCU_BWD_DATA, plan, count, alpha, dy, w, beta, dx, ws, ws_bytes, stream);
}

extern "C" mucu_status_t mucu_conv_backward_filter(mucu_handle_t h, const mucu_conv_desc_t* d,
                                                   const mucu_micro_config_t* plan, int32_t count, float alpha,
                                                   const void* x, const void* dy, float beta, float* dw, void* ws,
                                                   uint64_t ws_bytes, void* stream) {
    return execute(h, d, MUCU_BWD_FILTER, plan, count, alpha, x, dy, beta, dw, ws, ws_bytes, stream);
}

extern "C" mucu_status_t mucu_conv_backward_filter_reduce(mucu_handle_t h, const mucu_conv_desc_t* d,
                                                          const mucu_micro_config_t* plan, int32_t count, float alpha,
                                                          const void* x, const void* dy, float beta, float* dw,
                                                          const mucu_reduce_target_t* target, void* ws,
                                                          uint64_t ws_bytes, void* stream) {
    if (!target || target->count < 1 || target->count > MUCU_MAX_REDUCE_RANKS ||
        (target->multicast && target->count != 1))
        return set_error(MUCU_ERR_INVALID_VALUE, "reduce target: count must be 1..%d (1 for multicast)",
                         MUCU_MAX_REDUCE_RANKS);
    RedTarget red = {};
    for (int r = 0; r < target->count; ++r) {
        if (!target->dst[r] || ((uintptr_t)target->dst[r] & 15))
            return set_error(MUCU_ERR_MISALIGNED, "reduce target %d NULL or not 16-byte aligned", r);
        red.dst[r] = target->dst[r];
    }
    red.n = target->count;
    red.mc = target->multicast ? 1 : 0;
    return execute(h, d, MUCU_BWD_FILTER, plan, count, alpha, x, dy, beta, dw, ws, ws_bytes, stream, &red);
}

// ============================================================ benchmark ====
// Work per benchmark sample (ms): samples of longer micro-configurations use fewer launches.
constexpr float kBenchSampleMs = 1.0f;

static std::vector<int32_t> policy_sizes(int policy, int32_t n) {
    std::vector<int32_t> v;
    if (policy == MUCU_POLICY_ALL) {
        for (int32_t b = 1; b <= n; ++b) v.push_back(b);
    } else if (policy == MUCU_POLICY_POW2) {
        for (int32_t b = 1; b <= n; b *= 2) v.push_back(b);
        if (v.empty() || v.back() != n) v.push_back(n);  // reading G20
    } else {
        v.push_back(n);
    }
    return v;
}

struct ScratchLayout {
    uint64_t in0, in1, out, ws, total;
};

static ScratchLayout scratch_layout(const Geom& g, int type, uint64_t ws_limit) {
    const uint64_t elt = (uint64_t)elt_size(g.math);
    const uint64_t X = align_up((uint64_t)g.n * g.h * g.w * g.c * elt, 256);
    const uint64_t Y = align_up((uint64_t)g.n * g.p * g.q * g.k * elt, 256);
    const uint64_t Wt = align_up((uint64_t)g.k * g.r * g.s * g.c * elt, 256);
    const uint64_t DW = align_up((uint64_t)g.k * g.r * g.s * g.c * 4, 256);
    // Largest workspace any benchmarked micro-config may use.
    // ws grows with b, so min(ws(N), limit) bounds every b that fits the limit.
    uint64_t need = 0;
    for (int a = 0; a < MUCU_NUM_ALGOS; ++a) {
        WsLayout L;
        if (ws_layout(g, type, a, g.n, &L) == MUCU_OK) need = std::max(need, std::min(L.total, ws_limit));
    }
    need = align_up(need, 256);
    ScratchLayout s;
    s.in0 = 0;
    if (type == MUCU_FWD) { s.in1 = X; s.out = X + Wt; s.ws = X + Wt + Y; }
    else if (type == MUCU_BWD_DATA) { s.in1 = Y; s.out = Y + Wt; s.ws = Y + Wt + X; }
    else { s.in1 = X; s.out = X + Y; s.ws = X + Y + DW; }
    s.total = s.ws + need;
    return s;
}

extern "C" mucu_status_t mucu_benchmark_scratch_size(const mucu_conv_desc_t* d, mucu_conv_type_t type,
                                                     uint64_t ws_limit, uint64_t* bytes) {
    Geom g;
    if (!make_geom(d, &g) || !bytes || type < 0 || type > 2) return set_error(MUCU_ERR_INVALID_VALUE, "benchmark_scratch_size");
    *bytes = scratch_layout(g, type, ws_limit).total;
    return MUCU_OK;
}

static std::string cache_key(const mucu_conv_desc_t* d, int type, uint64_t limit, int policy, int warmup, int reps) {
    char buf[256];
    snprintf(buf, sizeof(buf), "%d,%d,%d,%d,%d,%d,%d,%d,%d,%d|%d|%llu|%d|%d|%d", d->n, d->c, d->h, d->w, d->k, d->r,
             d->s, d->pad, d->stride, d->math, type, (unsigned long long)limit, policy, warmup, reps);
    return buf;
}

extern "C" mucu_status_t mucu_benchmark(mucu_handle_t h, const mucu_conv_desc_t* d, mucu_conv_type_t type,
                                        uint64_t ws_limit, void* scratch, uint64_t scratch_bytes, void* stream,
                                        int64_t* time_ns, uint64_t* ws) {
    if (!h || !time_ns || !ws) return set_error(MUCU_ERR_INVALID_VALUE, "benchmark: bad arguments");
    Geom g;
    if (!make_geom(d, &g) || type < 0 || type > 2) return set_error(MUCU_ERR_INVALID_VALUE, "benchmark: invalid descriptor");
    const size_t cols = (size_t)g.n + 1;
    const std::string key = cache_key(d, type, ws_limit, h->policy, h->warmup, h->reps) + (h->deterministic ? "" : "|nd");
    auto it = h->cache.find(key);
    if (it != h->cache.end()) {  // P:L159 in-memory cache of benchmark results
        std::copy(it->second.first.begin(), it->second.first.end(), time_ns);
        std::copy(it->second.second.begin(), it->second.second.end(), ws);
        return MUCU_OK;
    }
    ScratchLayout S = scratch_layout(g, type, ws_limit);
    if (!scratch || scratch_bytes < S.total)
        return set_error(MUCU_ERR_INSUFFICIENT_WORKSPACE, "benchmark scratch %llu < %llu", (unsigned long long)scratch_bytes, (unsigned long long)S.total);
    if ((uintptr_t)scratch % 256) return set_error(MUCU_ERR_MISALIGNED, "scratch not 256-byte aligned");
    for (size_t i = 0; i < MUCU_NUM_ALGOS * cols; ++i) { time_ns[i] = -1; ws[i] = 0; }
    cudaStream_t st = (cudaStream_t)stream;
    char* base = (char*)scratch;
    cudaEvent_t e0, e1;
    if (cudaEventCreate(&e0) || cudaEventCreate(&e1)) return cuda_error((int)cudaGetLastError(), "event create");
    mucu_status_t status = MUCU_OK;
    std::vector<float> samples;
    for (int32_t b : policy_sizes(h->policy, g.n)) {
        for (int a = 0; a < MUCU_NUM_ALGOS && status == MUCU_OK; ++a) {
            WsLayout L;
            if (ws_layout(g, type, a, b, &L) != MUCU_OK || L.total > ws_limit) continue;
            // Steady state of a micro-batch inside a call: the b-independent prefix (padded /
            // space-to-depth filter, Winograd U, FFT filter spectrum) is computed once per
            // call by the executor, so the warm-up computes it and the timed runs reuse it.
            CallCtx bctx;
            auto launch = [&]() {
                return run_micro(h, g, type, a, b, 1.f, base + S.in0, base + S.in1, 0.f, base + S.out, base + S.ws,
                                 S.total - S.ws, st, &bctx);
            };
            // a dry run first: a configuration without a tensor-core kernel is skipped
            // (not benchmarked) whatever the warm-up count
            if (tc_math(g.math)) {
                CallCtx dry;
                dry.dry = true;
                if (run_micro(h, g, type, a, b, 1.f, base + S.in0, base + S.in1, 0.f, base + S.out, base + S.ws,
                              S.total - S.ws, st, &dry) == MUCU_ERR_UNSUPPORTED)
                    continue;
            }
            mucu_status_t r = MUCU_OK;
            // warm-up (the first launch builds the call's prefix); the last warm-up launch
            // is timed to size the samples
            float t1 = 0.f;
            for (int i = 0; i < h->warmup && r == MUCU_OK; ++i) {
                const bool last = i == h->warmup - 1;
                if (last) cudaEventRecord(e0, st);
                r = launch();
                if (last && r == MUCU_OK) {
                    cudaEventRecord(e1, st);
                    if (cudaEventSynchronize(e1)) { r = cuda_error((int)cudaGetLastError(), "benchmark sync"); break; }
                    cudaEventElapsedTime(&t1, e0, e1);
                }
            }
            if (r == MUCU_ERR_UNSUPPORTED) continue;
            if (r) { status = r; break; }
            // T_mu(b) (P:L88 step 1): micro-batches run back to back in a plan, so each sample
            // is the mean of `reps` back-to-back launches between two events (no idle-stream
            // launch latency in the table); the median of three samples is recorded.  A
            // sample needs no more launches than make ~1 ms of work (long micro-configs:
            // one launch per sample), which keeps the `all` policy's pass short.
            int reps = h->reps;
            if (t1 > 0.f) reps = std::max(1, std::min(h->reps, (int)std::ceil(kBenchSampleMs / t1)));
            samples.clear();
            for (int grp = 0; grp < 3 && r == MUCU_OK; ++grp) {
                cudaEventRecord(e0, st);
                for (int i = 0; i < reps && r == MUCU_OK; ++i) r = launch();
                cudaEventRecord(e1, st);
                if (r) break;
                if (cudaEventSynchronize(e1)) { r = cuda_error((int)cudaGetLastError(), "benchmark sync"); break; }
                float ms = 0.f;
                cudaEventElapsedTime(&ms, e0, e1);
                samples.push_back(ms / (float)reps);
            }
            if (r == MUCU_ERR_UNSUPPORTED) continue;
            if (r) { status = r; break; }
            std::sort(samples.begin(), samples.end());
            float med = samples[samples.size() / 2];
            time_ns[(size_t)a * cols + b] = (int64_t)(med * 1.0e6f + 0.5f);
            ws[(size_t)a * cols + b] = L.total;
        }
        if (status) break;
    }
    cudaEventDestroy(e0);
    cudaEventDestroy(e1);
    if (status) return status;
    int e = (int)cudaStreamSynchronize(st);
    if (e) return cuda_error(e, "benchmark stream");
    h->cache[key] = {std::vector<int64_t>(time_ns, time_ns + MUCU_NUM_ALGOS * cols),
                     std::vector<uint64_t>(ws, ws + MUCU_NUM_ALGOS * cols)};
    return MUCU_OK;
}

extern "C" mucu_status_t mucu_plan_layer(mucu_handle_t h, const mucu_conv_desc_t* d, mucu_conv_type_t type,
                                         uint64_t ws_limit, void* scratch, uint64_t scratch_bytes, void* stream,
                                         mucu_micro_config_t* out, int32_t cap, int32_t* count, int64_t* total_ns) {
    Geom g;
    if (!make_geom(d, &g)) return set_error(MUCU_ERR_INVALID_VALUE, "plan_layer: invalid descriptor");
    std::vector<int64_t> t((size_t)MUCU_NUM_ALGOS * (g.n + 1));
    std::vector<uint64_t> w(t.size());
    mucu_status_t s = mucu_benchmark(h, d, type, ws_limit, scratch, scratch_bytes, stream, t.data(), w.data());
    if (s) return s;
    return mucu_plan_wr(g.n, t.data(), w.data(), ws_limit, out, cap, count, total_ns);
}

// =================================================================== WD ====
extern "C" mucu_status_t mucu_network_create(mucu_network_t* net) {
    if (!net) return set_error(MUCU_ERR_INVALID_VALUE, "network_create");
    *net = new (std::nothrow) mucu_network();
    return *net ? MUCU_OK : set_error(MUCU_ERR_INTERNAL, "network_create: out of memory");
}

extern "C" mucu_status_t mucu_network_destroy(mucu_network_t net) {
    delete net;
    return MUCU_OK;
}

extern "C" mucu_status_t mucu_network_add(mucu_network_t net, const mucu_conv_desc_t* d, mucu_conv_type_t type,
                                          int32_t* kernel_id) {
    Geom g;
    if (!net || !make_geom(d, &g) || type < 0 || type > 2) return set_error(MUCU_ERR_INVALID_VALUE, "network_add");
    mucu_network::Kernel k;
    k.desc = *d;
    k.type = type;
    net->kernels.push_back(k);
    net->planned = false;
    if (kernel_id) *kernel_id = (int32_t)net->kernels.size() - 1;
    return MUCU_OK;
}

// Fronts (set-valued DP) per kernel, then the MCKP.
static mucu_status_t plan_network_tables(mucu_network_t net, uint64_t total_limit,
                                         const std::vector<std::vector<int64_t>>& T,
                                         const std::vector<std::vector<uint64_t>>& W) {
    const int K = (int)net->kernels.size();
    std::vector<std::vector<int64_t>> ft(K);
    std::vector<std::vector<uint64_t>> fm(K);
    std::vector<std::vector<std::vector<mucu_micro_config_t>>> fp(K);
    std::map<std::string, int> dedupe;  // identical (desc, type) share one front
    for (int k = 0; k < K; ++k) {
        const auto& kd = net->kernels[k];
        const int32_t n = kd.desc.n;
        std::string key = cache_key(&kd.desc, kd.type, total_limit, 0, 0, 0);
        auto it = dedupe.find(key);
        if (it != dedupe.end() && T[k] == T[it->second] && W[k] == W[it->second]) {
            ft[k] = ft[it->second]; fm[k] = fm[it->second]; fp[k] = fp[it->second];
            continue;
        }
        int32_t len = 0;
        mucu_status_t s = mucu_pareto_front(n, T[k].data(), W[k].data(), total_limit, nullptr, nullptr, 0, &len,
                                            nullptr, nullptr);
        if (s != MUCU_OK && s != MUCU_ERR_CAPACITY) return s == MUCU_ERR_INSUFFICIENT_WORKSPACE ? set_error(MUCU_ERR_INFEASIBLE, "kernel %d: nothing fits the total limit", k) : s;
        ft[k].resize(len); fm[k].resize(len);
        std::vector<mucu_micro_config_t> plans((size_t)len * n);
        std::vector<int32_t> plen(len);
        s = mucu_pareto_front(n, T[k].data(), W[k].data(), total_limit, ft[k].data(), fm[k].data(), len, &len,
                              plans.data(), plen.data());
        if (s) return s;
        fp[k].resize(len);
        for (int i = 0; i < len; ++i)
            fp[k][i].assign(plans.begin() + (size_t)i * n, plans.begin() + (size_t)i * n + plen[i]);
        dedupe[key] = k;
    }
    std::vector<int32_t> flen(K);
    std::vector<int64_t> tt;
    std::vector<uint64_t> mm;
    for (int k = 0; k < K; ++k) {
        flen[k] = (int32_t)ft[k].size();
        tt.insert(tt.end(), ft[k].begin(), ft[k].end());
        mm.insert(mm.end(), fm[k].begin(), fm[k].end());
    }
    std::vector<int32_t> choice(K);
    std::vector<uint64_t> offs(K);
    int64_t total = 0;
    mucu_status_t s = mucu_solve_wd(K, flen.data(), tt.data(), mm.data(), total_limit, choice.data(), offs.data(), &total);
    if (s) return s;
    for (int k = 0; k < K; ++k) {
        auto& kd = net->kernels[k];
        kd.plan = fp[k][choice[k]];
        kd.offset = offs[k];
        kd.bytes = align_up(fm[k][choice[k]], 256);
        kd.time_ns = ft[k][choice[k]];
    }
    net->planned = true;
    return MUCU_OK;
}

extern "C" mucu_status_t mucu_network_plan(mucu_network_t net, mucu_handle_t h, uint64_t total_limit, void* scratch,
                                           uint64_t scratch_bytes, void* stream) {
    if (!net || !h || net->kernels.empty()) return set_error(MUCU_ERR_INVALID_VALUE, "network_plan");
    const int K = (int)net->kernels.size();
    std::vector<std::vector<int64_t>> T(K);
    std::vector<std::vector<uint64_t>> W(K);
    for (int k = 0; k < K; ++k) {
        const auto& kd = net->kernels[k];
        const size_t sz = (size_t)MUCU_NUM_ALGOS * (kd.desc.n + 1);
        T[k].resize(sz); W[k].resize(sz);
        // A kernel can use at most the whole budget; the cache dedupes repeats.
        mucu_status_t s = mucu_benchmark(h, &kd.desc, (mucu_conv_type_t)kd.type, total_limit, scratch, scratch_bytes,
                                         stream, T[k].data(), W[k].data());
        if (s) return s;
    }
    return plan_network_tables(net, total_limit, T, W);
}

extern "C" mucu_status_t mucu_network_plan_from_tables(mucu_network_t net, uint64_t total_limit, const int64_t* time_ns,
                                                       const uint64_t* ws) {
    if (!net || net->kernels.empty() || !time_ns || !ws) return set_error(MUCU_ERR_INVALID_VALUE, "network_plan_from_tables");
    const int K = (int)net->kernels.size();
    std::vector<std::vector<int64_t>> T(K);
    std::vector<std::vector<uint64_t>> W(K);
    size_t off = 0;
    for (int k = 0; k < K; ++k) {
        const size_t sz = (size_t)MUCU_NUM_ALGOS * (net->kernels[k].desc.n + 1);
        T[k].assign(time_ns + off, time_ns + off + sz);
        W[k].assign(ws + off, ws + off + sz);
        off += sz;
    }
    return plan_network_tables(net, total_limit, T, W);
}

extern "C" mucu_status_t mucu_network_get(mucu_network_t net, int32_t kernel_id, mucu_micro_config_t* out, int32_t cap,
                                          int32_t* count, uint64_t* ws_offset, uint64_t* ws_bytes, int64_t* time_ns) {
    if (!net || kernel_id < 0 || kernel_id >= (int32_t)net->kernels.size() || !count)
        return set_error(MUCU_ERR_INVALID_VALUE, "network_get");
    if (!net->planned) return set_error(MUCU_ERR_INVALID_VALUE, "network_get: network not planned");
    const auto& kd = net->kernels[kernel_id];
    *count = (int32_t)kd.plan.size();
    if (ws_offset) *ws_offset = kd.offset;
    if (ws_bytes) *ws_bytes = kd.bytes;
    if (time_ns) *time_ns = kd.time_ns;
    if (!out || cap < *count) return set_error(MUCU_ERR_CAPACITY, "network_get: capacity");
    std::copy(kd.plan.begin(), kd.plan.end(), out);
    return MUCU_OK;
}
