// tc_gemm_kernel.cuh -- the persistent tcgen05 conv-GEMM kernel (included by
// kernels_tc.cu inside namespace mucu::{anon}; see the file header there).
//
// Persistent CTAs (grid = min(tiles, #SMs)) walk the output tiles
// (m fastest, then n, then batch / split z).  Warp roles, 288 threads:
//   warps 0-3  producers: one thread issues TMA (tiled or im2col mode), all 128
//              gather with cp.async / st.shared where TMA cannot express the
//              operand; the smem ring runs continuously across tiles;
//   warp  4    TMEM allocator + single-thread tcgen05.mma issuer;
//   warps 5-8  epilogue (TMEM lane quadrant = warp % 4).
// Two TMEM accumulators (2 x BN columns) let the epilogue of tile i overlap
// the mainloop of tile i+1 (tmem_full / tmem_empty barriers).

// Ticket counter of this launch (value (epoch << 20) + tickets taken; a value of an
// older launch counts as 0): returns this caller's ticket 0, 1, 2, ...
__device__ __forceinline__ int take_ticket(unsigned long long* c, unsigned long long epoch) {
    unsigned long long old = *(volatile unsigned long long*)c;
    for (;;) {
        const bool fresh = (old >> 20) == epoch;
        const unsigned long long want = fresh ? old + 1 : (epoch << 20) + 1;
        const unsigned long long prev = atomicCAS(c, old, want);
        if (prev == old) return fresh ? (int)(old & 0xFFFFFull) : 0;
        old = prev;
    }
}

// dw element (offset from the batch's dw base) of BackwardFilter GEMM element
// (row m, column n) for each split-K epilogue layout; -1 = padding (no element).
template <int EPI, int ELT>
__device__ __forceinline__ long long wgrad_dst(const TcArgs& p, int m, int n) {
    if constexpr (EPI == EPI_WGRAD_CHAIN) {
        return (long long)m * p.ldc + n;
    } else if constexpr (EPI == EPI_WGRAD_SMALLC) {
        // padded column j' = (r, s8, c') -> dw column (r*S + s)*C + c
        const int c = n % p.cp, t2 = n / p.cp, s_ = t2 % p.s8, r = t2 / p.s8;
        return (c < p.C && s_ < p.S) ? (long long)m * p.ldc + (r * p.S + s_) * p.C + c : -1;
    } else if constexpr (EPI == EPI_WGRAD_S2D) {
        // column (tap (d,e), channel (a, b, c)) -> dw[k][st*d+a][st*e+b][c]
        const int stc = p.s2_st * p.s2_C, real = stc * p.s2_st;
        const int tap = n / p.C, ch = n - tap * p.C;
        if (ch >= real) return -1;
        const int d = tap / p.S, e = tap - d * p.S;
        const int a = ch / stc, rem = ch - a * stc, bq = rem / p.s2_C, c = rem - bq * p.s2_C;
        const int r = p.s2_st * d + a, sx = p.s2_st * e + bq;
        return (r < p.s2_R && sx < p.s2_S) ? (long long)m * p.ldc + (r * p.s2_S + sx) * p.s2_C + c : -1;
    } else if constexpr (EPI == EPI_WGRAD_TAPS) {
        return m < p.kred_taps ? (long long)n * p.ldc + m : -1;
    } else if constexpr (EPI == EPI_WGRAD_WIN) {
        // row m = (r, atom aa, tap t, channel c) -> dw[k = n][r][aa*taps + t][c]
        const int per_atom = p.win_aw / ELT;  // elements per A swizzle atom
        const int ja = m / per_atom, e = m - ja * per_atom;
        const int t = e / p.cp, c = e - t * p.cp;
        const int r = ja / p.win_na, sx = (ja - r * p.win_na) * (per_atom / p.cp) + t;
        return (r < p.R && sx < p.S && c < p.C) ? (long long)n * p.ldc + (r * p.S + sx) * p.C + c : -1;
    } else {
        return -1;
    }
}

// dst[ofs[j] * stride] = alpha * v[j] + beta * dst[...] for the 32 accumulator
// columns of one row (ofs < 0: skipped); all loads issue before the stores.
// beta == 0 never reads dst (it may hold garbage / NaN).
// red (NEXT-3): the cross-rank dW sum (nullptr: off); red_off = element offset of dst in
// dw -- the final value of every element is also added there.
__device__ __forceinline__ void rmw32(float* dst, const int (&ofs)[32], size_t stride, const uint32_t* v, float alpha,
                                      float beta, bool atomic = false, const RedTarget* red = nullptr,
                                      long long red_off = 0) {
    if (atomic) {  // non-deterministic split-K (beta applied by a prescale launch): L2 reductions
#pragma unroll
        for (int j = 0; j < 32; ++j)
            if (ofs[j] >= 0)
                asm volatile("red.global.add.f32 [%0], %1;" ::"l"(dst + (size_t)ofs[j] * stride),
                             "f"(alpha * __uint_as_float(v[j]))
                             : "memory");
        return;
    }
    float old[32];
#pragma unroll
    for (int j = 0; j < 32; ++j) old[j] = (beta != 0.f && ofs[j] >= 0) ? __ldcg(dst + (size_t)ofs[j] * stride) : 0.f;
#pragma unroll
    for (int j = 0; j < 32; ++j)
        if (ofs[j] >= 0) {
            const float o = alpha * __uint_as_float(v[j]) + beta * old[j];
            dst[(size_t)ofs[j] * stride] = o;
            if (red) red_add(*red, red_off + (long long)ofs[j] * (long long)stride, o);
        }
}

template <int ELT, int AM, int BM_, int EPI>
__global__ void __launch_bounds__(threads_for(AM), 1) tc_conv_gemm(const __grid_constant__ TcArgs p,
                                                            const __grid_constant__ CUtensorMap tmA,
                                                            const __grid_constant__ CUtensorMap tmB) {
    using T = typename Elt<ELT>::T;
    constexpr int KB = 128 / ELT;            // K elements per stage
    constexpr int UMMA_K = 32 / ELT;         // K elements per MMA
    // p.mt blocks of 128 rows x 128 B (tile M = 128 * p.mt); MN-major WGRAD
    // stages hold p.km k-blocks (p.km x KB rows of K per 128-B atom column).
    const int A_HALF = 128 * 128 * p.km;
    constexpr bool HALO = (AM == A_HALO);
    const int A_BYTES = HALO ? 0 : p.mt * A_HALF;
    const int KD = KB * p.km;                // K rows per stage (MN-major modes)
    constexpr bool WIN = (AM == A_TMA_WIN || AM == A_TMA_WIN64 || AM == A_TMA_WIN32);
    constexpr uint32_t WAW = AM == A_TMA_WIN64 ? 64u : AM == A_TMA_WIN32 ? 32u : 128u;  // window atom bytes
    // A_STAGED_WG: small-C strided BackwardFilter, zero workspace: x rows staged by TMA,
    // the exact-tap MN-major A operand (rows = (r,s,c), K = output pixels) built in
    // shared memory by 256 builder threads (warps 0-3 and 5-8)
    constexpr bool STAGED = (AM == A_STAGED_WG);
    // A_STAGED_FWD: small-C strided forward, zero workspace (x rows staged by TMA, the
    // exact-tap K-major A operand built in shared memory, the filter resident)
    constexpr bool STAGED_FWD = (AM == A_STAGED_FWD);
    constexpr bool A_MN = (AM == A_TMA_MN2 || WIN || STAGED);
    constexpr bool B_MN = (BM_ == B_TMA_MN2 || BM_ == B_TMA_MN3 || BM_ == B_GATHER_WG || BM_ == B_SCALAR_DGRAD ||
                           BM_ == B_SCALAR_WG || BM_ == B_TMA_IM2COL || BM_ == B_GATHER_SMALLC ||
                           BM_ == B_GATHER_SMALLC_PAD || BM_ == B_TMA_DYROW);
    constexpr bool A_TMA = (AM == A_TMA_K2 || AM == A_TMA_K3 || AM == A_TMA_MN2 || AM == A_TMA_IM2COL || WIN ||
                            AM == A_HALO);
    constexpr bool B_TMA = (BM_ == B_TMA_K2 || BM_ == B_TMA_K3 || BM_ == B_TMA_MN2 || BM_ == B_TMA_MN3 ||
                            BM_ == B_TMA_IM2COL || BM_ == B_TMA_DYROW);
    constexpr bool B_RES = (BM_ == B_RESIDENT);  // (A_STAGED_FWD stages the filter at sB)
    constexpr bool GATHER = !A_TMA || (!B_TMA && !B_RES);
    constexpr bool SPLITK = (EPI == EPI_WGRAD_CHAIN || EPI == EPI_WGRAD_SMALLC || EPI == EPI_WGRAD_S2D ||
                             EPI == EPI_WGRAD_WIN || EPI == EPI_WGRAD_TAPS || EPI == EPI_WGRAD_PARTIAL);
    constexpr bool A_ASYNC = (AM == A_GATHER_FWD || AM == A_GATHER_DGRAD || AM == A_GATHER_SMALLC_PAD);
    constexpr bool B_ASYNC = (BM_ == B_GATHER_WG || BM_ == B_GATHER_SMALLC_PAD);
    // MN-major atoms: 8-row (bf16, SWIZZLE_128B) or 4-row (tf32, 128B_BASE32B) groups.
    constexpr uint32_t MN_SBO = ELT == 2 ? 1024u : 512u;
    constexpr uint32_t MN_LAYOUT = ELT == 2 ? 2u : 1u;
    constexpr bool WALK = (AM == A_GATHER_FWD || AM == A_GATHER_DGRAD || AM == A_TMA_IM2COL);

    extern __shared__ uint8_t smem_raw[];
    uint8_t* smem = (uint8_t*)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
    const int S = p.stages;
    const int B_BYTES = p.b_bytes * p.km;
    uint8_t* sA = smem;
    // A_HALO: a ring of p.hstages halo tiles (p.halo_bytes each) replaces the A stages
    uint8_t* sB = smem + (HALO ? (size_t)p.hstages * p.halo_bytes : (size_t)S * A_BYTES);
    uint8_t* sBres = sB + (size_t)S * B_BYTES;  // B_RESIDENT: whole filter, k-block after k-block
    // cluster split-K: the epilogue stages the partial tile over the operand ring, so
    // the barriers sit past whichever region is larger
    uint8_t* bar_base = sBres + p.bres_bytes;  // B_RESIDENT filter / A_STAGED_WG x ring + tap table
    if (smem + p.stg_bytes > bar_base) bar_base = smem + p.stg_bytes;
    uint64_t* bars = (uint64_t*)bar_base;
    uint64_t* full = bars;
    uint64_t* empty = bars + S;
    uint64_t* tfull = bars + 2 * S;      // [2]
    uint64_t* tempty = bars + 2 * S + 2; // [2]
    uint64_t* bres_bar = bars + 2 * S + 4;
    uint32_t* tmem_slot = (uint32_t*)(bars + 2 * S + 5);
    uint64_t* hfull = bars + 2 * S + 6;             // [hstages] halo ring
    uint64_t* hempty = bars + 2 * S + 6 + p.hstages;
    uint64_t* xfull = bars + 2 * S + 6 + 2 * p.hstages;               // [sx_stages] staged x rows
    uint64_t* xempty = bars + 2 * S + 6 + 2 * p.hstages + p.sx_stages;

    const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
    const int BMt = 128 * p.mt;  // tile rows: 128, or 256 as two 128-row halves with separate accumulators
    const int mt = (p.M + BMt - 1) / BMt, nt = (p.N + p.BN - 1) / p.BN;
    const int per_z = mt * nt;
    const int total_tiles = per_z * p.num_z;

    if (threadIdx.x == 0) {
        const uint32_t full_count = STAGED ? 257u : STAGED_FWD ? 128u : (GATHER ? 128u : 0u) + (A_TMA || B_TMA ? 1u : 0u);
        for (int s = 0; s < S; ++s) {
            mbar_init(smem_u32(&full[s]), full_count);
            mbar_init(smem_u32(&empty[s]), 1);
        }
        for (int a = 0; a < 2; ++a) {
            mbar_init(smem_u32(&tfull[a]), 1);
            mbar_init(smem_u32(&tempty[a]), 4);
        }
        mbar_init(smem_u32(bres_bar), 128);
        for (int h = 0; h < p.hstages; ++h) {
            mbar_init(smem_u32(&hfull[h]), 1);
            mbar_init(smem_u32(&hempty[h]), 1);
        }
        for (int j = 0; j < p.sx_stages; ++j) {
            mbar_init(smem_u32(&xfull[j]), 1);
            mbar_init(smem_u32(&xempty[j]), STAGED ? 256 : 128);
        }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    if (warp == 4) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(tmem_slot)),
                     "r"(p.tmem_cols));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tmem = *tmem_slot;
    // Programmatic dependent launch: the prologue above (barrier init, TMEM
    // allocation) overlaps the previous kernel's tail; wait for its results
    // before the first global access, then let the next launch start its own.
    asm volatile("griddepcontrol.wait;" ::: "memory");
    asm volatile("griddepcontrol.launch_dependents;" :::);

    // Cluster split-K with ordered split groups: a cluster's group (= which k-range of
    // its tile it reduces, and its place in the tile's addition order) is a ticket
    // taken when the cluster starts, not its cluster id, so a group only ever waits
    // for groups that were already running -- no dependency on the scheduling order
    // of clusters (GPC packing, concurrent kernels).  The k-range of group g is fixed,
    // so the summation order, and dw, do not depend on which cluster got which ticket.
    // "Running" means every CTA of the cluster holds its tensor memory: the ticket is
    // taken only after a cluster barrier behind all ranks' tcgen05.alloc.  (A rank
    // still blocked in the allocation -- its SM's TMEM held by a co-resident CTA that
    // waits on a later group -- would otherwise deadlock behind its own ticket.)
    int g_ticket = -1;
    if constexpr (SPLITK) {
        if (p.cl && p.tickets) {
            int& s_tk = ((int*)tmem_slot)[1];  // (dynamic shared memory: the upper half of the TMEM slot)
            const int rho = blockIdx.x % p.cl, c = blockIdx.x / p.cl;
            const int nu = per_z * (p.zsplit ? p.num_z / p.zsplit : 1);
            asm volatile("barrier.cluster.arrive.release;\n\tbarrier.cluster.wait.acquire;" ::: "memory");
            if (threadIdx.x == 0 && rho == 0) s_tk = take_ticket(p.tickets + (c % nu), p.epoch);
            asm volatile("barrier.cluster.arrive.release;\n\tbarrier.cluster.wait.acquire;" ::: "memory");
            if (threadIdx.x == 0 && rho != 0) {
                uint32_t ra;
                asm("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(ra) : "r"(smem_u32(&s_tk)), "r"(0));
                int v;
                asm volatile("ld.shared::cluster.s32 %0, [%1];" : "=r"(v) : "r"(ra) : "memory");
                s_tk = v;
            }
            __syncthreads();
            g_ticket = s_tk;
            // rank 0 may not leave (and drop its shared memory) before the others read it
            asm volatile("barrier.cluster.arrive.release;\n\tbarrier.cluster.wait.acquire;" ::: "memory");
        }
    }

    // tile -> (m0, n0, z, k-block range)
    // Cluster split-K (p.cl > 0, one unit per CTA): CTA `tile` is rank tile % cl of
    // cluster c = tile / cl; cluster c = (split group g, batch, output tile), g
    // slowest; split = g * cl + rank.
    auto decode = [&](int tile, int& m0, int& n0, int& z, int& kb_begin, int& kb_end) {
        int rem;
        if (p.cl) {
            const int rho = tile % p.cl, c = tile / p.cl;
            const int nbatch = p.zsplit ? p.num_z / p.zsplit : 1;
            const int nu = per_z * nbatch;
            const int g = g_ticket >= 0 ? g_ticket : c / nu, u = c % nu;
            const int batch = u / per_z;
            rem = u - batch * per_z;
            const int split = g * p.cl + rho;
            z = p.zsplit ? batch * p.zsplit + split : split;
        } else {
            z = tile / per_z;
            rem = tile - z * per_z;
        }
        const int ntile = rem / mt;
        m0 = (rem - ntile * mt) * BMt;
        n0 = ntile * p.BN;
        kb_begin = 0; kb_end = p.ph_n ? p.ph_kbv[z] : p.num_kb;
        if (SPLITK) {
            // batched split-K (Winograd BackwardFilter): z = batch * zsplit + split
            const int sp = p.zsplit ? z % p.zsplit : z;
            kb_begin = sp * p.kb_per_split;
            kb_end = min(p.num_kb, kb_begin + p.kb_per_split);
        }
    };

    if constexpr (STAGED) {
        // ================= staged-row producers (A_STAGED_WG) =================
        // k-block kb = KD output pixels (n, p, q0 .. q0+KD-1) of output row n*P + p;
        // x rows st*p + r - pad (r < R), elements [chunk0*cs, (chunk0 + bch)*cs) of each
        // row (zero outside the image) land in an x stage by one TMA box; GEMM row
        // m = (r, s, c) of pixel q reads staged[r][tab(m) + col0 + st*C*(q - q0)].
        // Warp 9 issues the x and dy TMA loads (running ahead over an sx_stages ring);
        // warps 0-3 and 5-8 (256 threads) build the A operand.  Each builder owns fixed
        // work units (a 16-B chunk of the tap axis x 4 consecutive pixels) whose
        // shared-memory source offsets and swizzled destinations are computed once.
        int* tab = (int*)(sBres + (size_t)p.sx_stages * p.sx_bytes);
        const int TR = 128 * p.mt;
        constexpr int EPC = 16 / ELT;             // elements per 16-B chunk
        const int CH = TR / EPC;                  // chunks per A K-row (pixel)
        const int stC = p.stride * p.C;
        // k-block walk: (output row n*P + p, q-block qb) -> the x stage's TMA coordinates
        // and the builders' column offset.  Divisions once per tile (init), then each
        // k-block advances incrementally (the builders' integer divisions were a third
        // of their stall samples).
        struct XWalk {
            int qb, pp, n_, chunk0, col0, cq0;
            int chunk_start, col_start, adv_q, adv_r;
        };
        auto x_init = [&](int kb, XWalk& w) {
            const int row = kb / p.win_qb;
            w.qb = kb - row * p.win_qb;
            w.n_ = row / p.P;
            w.pp = row - w.n_ * p.P;
            const int e_start = -p.pad * p.C;  // e0 of q-block 0
            w.chunk_start = e_start >= 0 ? e_start / p.sx_cs : -((-e_start + p.sx_cs - 1) / p.sx_cs);
            w.col_start = e_start - w.chunk_start * p.sx_cs;
            const int adv = p.stride * KD * p.C;  // e0 step per q-block
            w.adv_q = adv / p.sx_cs;
            w.adv_r = adv - w.adv_q * p.sx_cs;
            w.cq0 = w.qb * KD;
            const int e0 = (p.stride * w.cq0 - p.pad) * p.C;
            w.chunk0 = e0 >= 0 ? e0 / p.sx_cs : -((-e0 + p.sx_cs - 1) / p.sx_cs);
            w.col0 = e0 - w.chunk0 * p.sx_cs;
        };
        auto x_step = [&](XWalk& w) {
            if (++w.qb == p.win_qb) {
                w.qb = 0; w.cq0 = 0; w.chunk0 = w.chunk_start; w.col0 = w.col_start;
                if (++w.pp == p.P) { w.pp = 0; ++w.n_; }
            } else {
                w.cq0 += KD;
                w.chunk0 += w.adv_q;
                w.col0 += w.adv_r;
                if (w.col0 >= p.sx_cs) { w.col0 -= p.sx_cs; ++w.chunk0; }
            }
        };
        if (warp == 9) {
            if (lane == 0) {
                int s = 0, jx = 0;
                uint32_t ph = 0, xph = 0;
                for (int tile = blockIdx.x; tile < total_tiles; tile += gridDim.x) {
                    int m0, n0, z, kb_begin, kb_end;
                    decode(tile, m0, n0, z, kb_begin, kb_end);
                    XWalk w;
                    if (kb_begin < kb_end) x_init(kb_begin, w);
                    for (int kb = kb_begin; kb < kb_end; ++kb) {
                        // x rows into ring stage jx (freed by the builders)
                        mbar_wait(smem_u32(&xempty[jx]), xph ^ 1u);
                        const uint32_t xb = smem_u32(&xfull[jx]);
                        mbar_arrive_tx(xb, (uint32_t)p.sx_tx);
                        tma_load_4d(smem_u32(sBres + (size_t)jx * p.sx_bytes), &tmA, xb, 0, w.chunk0,
                                    p.stride * w.pp - p.pad, w.n_);
                        // dy of the KD pixels into operand stage s (freed by the MMA)
                        mbar_wait(smem_u32(&empty[s]), ph ^ 1u);
                        const uint32_t bT = smem_u32(sB + (size_t)s * B_BYTES);
                        const uint32_t fb = smem_u32(&full[s]);
                        mbar_arrive_tx(fb, (uint32_t)p.tma_bytes);
                        const int row = w.n_ * p.P + w.pp;
                        for (int a = 0; a < p.bn_atoms; ++a)
                            tma_load_3d(bT + a * KD * 128, &tmB, fb, n0 + a * (128 / ELT), w.cq0, row);
                        x_step(w);
                        if (++s == S) { s = 0; ph ^= 1u; }
                        if (++jx == p.sx_stages) { jx = 0; xph ^= 1u; }
                    }
                }
            }
            __syncwarp();
        } else if (warp != 4) {
            const int bt = warp < 4 ? threadIdx.x : threadIdx.x - 32;  // 0..255
            for (int m = bt; m < TR; m += 256) tab[m] = m < p.kred_taps ? (m / (p.S * p.C)) * p.sx_sr + m % (p.S * p.C) : -1;
            asm volatile("bar.sync 2, 256;" ::: "memory");
            // this thread's units u = bt + 256 j: chunk ch = u % CH, pixel group gr = u / CH
            constexpr int MAXU = 4;
            const int ngr_all = KD / 4, nunits = CH * ngr_all;
            int u_gr[MAXU], u_src[MAXU][EPC];
            uint32_t u_dst[MAXU];
#pragma unroll
            for (int j = 0; j < MAXU; ++j) {
                const int u = bt + 256 * j;
                u_gr[j] = u < nunits ? u / CH : 1 << 20;
                const int ch = u - (u / CH) * CH, m0e = ch * EPC;
                const int hh = m0e >> 7, mi = m0e & 127;
                // destination of pixel row kr = 4*gr + rr: row base + swizzled chunk (the
                // swizzle depends on kr % 4 (tf32) / kr % 8 (bf16), i.e. on rr and gr)
                u_dst[j] = (uint32_t)(hh * A_HALF) + (uint32_t)((mi / (128 / ELT)) * KD * 128) +
                           mn_row_off<ELT>(4 * (u_gr[j] & 1), (mi % (128 / ELT)) * ELT) - 512u * (u_gr[j] & 1);
#pragma unroll
                for (int e = 0; e < EPC; ++e) {
                    const int t = u < nunits ? tab[m0e + e] : -1;
                    u_src[j][e] = t >= 0 ? (t + stC * 4 * u_gr[j]) * ELT : -1;
                }
            }
            int s = 0, jx = 0;
            uint32_t ph = 0, xph = 0;
            for (int tile = blockIdx.x; tile < total_tiles; tile += gridDim.x) {
                int m0, n0, z, kb_begin, kb_end;
                decode(tile, m0, n0, z, kb_begin, kb_end);
                XWalk w;
                if (kb_begin < kb_end) x_init(kb_begin, w);
                for (int kb = kb_begin; kb < kb_end; ++kb) {
                    const int valid = min(KD, p.Q - w.cq0);
                    mbar_wait(smem_u32(&empty[s]), ph ^ 1u);
                    mbar_wait(smem_u32(&xfull[jx]), xph);
                    const uint32_t aT = smem_u32(sA + (size_t)s * A_BYTES);
                    const uint32_t xs = smem_u32(sBres) + (uint32_t)(jx * p.sx_bytes) + (uint32_t)(w.col0 * ELT);
                    // rows (pixels) the MMA reads: valid rounded up to the MMA K step (the
                    // rest of the stage is never read; dy rows past Q are zero-filled)
                    const int nrows = min(KD, (valid + UMMA_K - 1) / UMMA_K * UMMA_K);
#pragma unroll
                    for (int j = 0; j < MAXU; ++j) {
                        if (4 * u_gr[j] >= nrows) continue;
#pragma unroll
                        for (int rr = 0; rr < 4; ++rr) {
                            const int kr = 4 * u_gr[j] + rr;
                            if (kr >= nrows) break;
                            const uint32_t xrow = xs + (uint32_t)(stC * rr * ELT);
                            uint32_t w[4];
                            if constexpr (ELT == 4) {
#pragma unroll
                                for (int e = 0; e < 4; ++e) {
                                    uint32_t v = 0u;
                                    if (u_src[j][e] >= 0)
                                        asm volatile("ld.shared.b32 %0, [%1];" : "=r"(v) : "r"(xrow + (uint32_t)u_src[j][e]));
                                    w[e] = v;
                                }
                            } else {
#pragma unroll
                                for (int e = 0; e < 4; ++e) {
                                    unsigned short lo = 0, hi = 0;
                                    if (u_src[j][2 * e] >= 0)
                                        asm volatile("ld.shared.u16 %0, [%1];" : "=h"(lo) : "r"(xrow + (uint32_t)u_src[j][2 * e]));
                                    if (u_src[j][2 * e + 1] >= 0)
                                        asm volatile("ld.shared.u16 %0, [%1];" : "=h"(hi) : "r"(xrow + (uint32_t)u_src[j][2 * e + 1]));
                                    w[e] = (uint32_t)lo | ((uint32_t)hi << 16);
                                }
                            }
                            // row kr: + kr * 128; the swizzle XOR of kr's low bits (rr) on the
                            // 16-B (bf16) / 32-B (tf32) chunk index
                            const uint32_t dst = aT + u_dst[j] + (uint32_t)(kr * 128);
                            const uint32_t sw = ELT == 4 ? ((uint32_t)(rr & 3) << 5) : ((uint32_t)(rr & 3) << 4);
                            asm volatile("st.shared.v4.b32 [%0], {%1, %2, %3, %4};" ::"r"(dst ^ sw), "r"(w[0]),
                                         "r"(w[1]), "r"(w[2]), "r"(w[3])
                                         : "memory");
                        }
                    }
                    fence_proxy_async();
                    mbar_arrive(smem_u32(&full[s]));
                    mbar_arrive(smem_u32(&xempty[jx]));
                    x_step(w);
                    if (++s == S) { s = 0; ph ^= 1u; }
                    if (++jx == p.sx_stages) { jx = 0; xph ^= 1u; }
                }
            }
        }
    }
    if constexpr (STAGED_FWD) {
        // ============== staged-row forward producers (A_STAGED_FWD) ==============
        // Tile = T output rows (p0 .. p0+T-1) of one image, GEMM row i = t*Q + q.  The
        // st*(T-1) + R x rows the tile reads are staged by TMA (one box per row) into a
        // buffer with zeroed left / right margins (the padding taps read zeros); the
        // K-major A operand (K = the exact (r, s, c) taps) is built from it per k-block;
        // the filter is staged once per CTA (B resident).  Warp 9 issues the TMA loads,
        // warps 0-3 (128 threads) build; the epilogue warps drain tiles meanwhile.
        const int Tr = p.win_qb;                     // output rows per tile
        const int XR = p.stride * (Tr - 1) + p.R;    // staged x rows per tile
        const int tiles_img = (p.P + Tr - 1) / Tr;
        const int xoff = p.sx_cs;                    // element offset of column 0 in a staged row
        uint8_t* sXr = sBres + p.sxw_off;            // x-row ring after the resident filter
        if (warp == 9) {
            if (lane == 0) {
                int ti = 0;
                for (int tile = blockIdx.x; tile < total_tiles; tile += gridDim.x, ++ti) {
                    const int jx = ti % p.sx_stages;
                    mbar_wait(smem_u32(&xempty[jx]), (uint32_t)(((ti / p.sx_stages) & 1) ^ 1));
                    const int n_ = tile / tiles_img, p0 = (tile - n_ * tiles_img) * Tr;
                    const uint32_t xb = smem_u32(&xfull[jx]);
                    mbar_arrive_tx(xb, (uint32_t)p.sx_tx);
                    const uint32_t dst = smem_u32(sXr + (size_t)jx * p.sx_bytes) + (uint32_t)(xoff * ELT);
                    for (int r = 0; r < XR; ++r)
                        tma_load_4d(dst + (uint32_t)(r * p.sx_sr * ELT), &tmA, xb, 0, 0, p.stride * p0 - p.pad + r, n_);
                }
            }
            __syncwarp();
        } else if (warp < 4) {
            const int bt = threadIdx.x;  // 0..127
            int* tab = (int*)(sXr + (size_t)p.sx_stages * p.sx_bytes);
            const uint32_t tab_s = smem_u32(tab);
            uint8_t* sW = sBres;                                         // resident filter, k-block by k-block
            const int KP = p.num_kb * KB;                                // taps padded to whole k-blocks
            // tap table: element offset of tap k = (r, s, c) relative to (row 0, column st*q - pad)
            for (int k = bt; k < KP; k += 128)
                tab[k] = k < p.kred_taps ? (k / (p.S * p.C)) * p.sx_sr + (k % (p.S * p.C)) - p.pad * p.C + xoff : -1;
            // zero the staged margins (TMA writes only the interior of each row)
            for (int j = 0; j < p.sx_stages; ++j)
                for (int e = bt; e < XR * p.sx_sr; e += 128) {
                    const int col = e % p.sx_sr;
                    if (col < xoff || col >= xoff + p.W * p.C) {
                        if constexpr (ELT == 4) ((float*)(sXr + (size_t)j * p.sx_bytes))[e] = 0.f;
                        else ((unsigned short*)(sXr + (size_t)j * p.sx_bytes))[e] = 0;
                    }
                }
            // resident filter B[n][k] = w[n][k] (k < R*S*C, else 0), K-major SW128 per k-block
            const T* wsrc = (const T*)p.bsrc;
            for (int idx = bt; idx < p.num_kb * p.BN * KB; idx += 128) {
                const int kb = idx / (p.BN * KB), rem = idx - kb * (p.BN * KB);
                const int n = rem / KB, e = rem - n * KB, k = kb * KB + e;
                const T v = (n < p.N && k < p.kred_taps) ? wsrc[(size_t)n * p.kred_taps + k] : (T)0.f;
                st_shared_elt<T>(smem_u32(sW) + (uint32_t)(kb * p.BN * 128) + kmaj_off(n, e * ELT), v);
            }
            fence_proxy_async();
            asm volatile("bar.sync 2, 128;" ::: "memory");
            mbar_arrive(smem_u32(bres_bar));
            // this thread: chunk c8 = bt % 8 (16 B of a k-block row), rows i = bt / 8 + 16 j
            const int c8 = bt & 7;
            constexpr int EPC = 16 / ELT;
            int ai = 0, ti = 0;
            for (int tile = blockIdx.x; tile < total_tiles; tile += gridDim.x, ++ti) {
                const int jx = ti % p.sx_stages;
                int rowoff[8];
#pragma unroll
                for (int j = 0; j < 8; ++j) {
                    const int i = bt / 8 + 16 * j, t = i / p.Q, q = i - t * p.Q;
                    rowoff[j] = t < Tr ? (p.stride * t * p.sx_sr + p.stride * q * p.C) * ELT : -1;
                }
                mbar_wait(smem_u32(&xfull[jx]), (uint32_t)((ti / p.sx_stages) & 1));
                const uint32_t xs = smem_u32(sXr) + (uint32_t)(jx * p.sx_bytes);
                for (int kb = 0; kb < p.num_kb; ++kb, ++ai) {
                    const int s = ai % S;
                    mbar_wait(smem_u32(&empty[s]), (uint32_t)(((ai / S) & 1) ^ 1));
                    int tv[EPC];
#pragma unroll
                    for (int e = 0; e < EPC; e += 4)
                        asm volatile("ld.shared.v4.s32 {%0, %1, %2, %3}, [%4];"
                                     : "=r"(tv[e]), "=r"(tv[e + 1]), "=r"(tv[e + 2]), "=r"(tv[e + 3])
                                     : "r"(tab_s + (uint32_t)((kb * KB + c8 * EPC + e) * 4)));
                    const uint32_t aT = smem_u32(sA + (size_t)s * A_BYTES);
#pragma unroll
                    for (int j = 0; j < 8; ++j) {
                        const int i = bt / 8 + 16 * j;
                        uint32_t w[4] = {0u, 0u, 0u, 0u};
                        if (rowoff[j] >= 0) {
                            const uint32_t xr = xs + (uint32_t)rowoff[j];
                            if constexpr (ELT == 4) {
#pragma unroll
                                for (int e = 0; e < 4; ++e)
                                    if (tv[e] >= 0)
                                        asm volatile("ld.shared.b32 %0, [%1];" : "=r"(w[e]) : "r"(xr + (uint32_t)(tv[e] * 4)));
                            } else {
#pragma unroll
                                for (int e = 0; e < 4; ++e) {
                                    unsigned short lo = 0, hi = 0;
                                    if (tv[2 * e] >= 0)
                                        asm volatile("ld.shared.u16 %0, [%1];" : "=h"(lo) : "r"(xr + (uint32_t)(tv[2 * e] * 2)));
                                    if (tv[2 * e + 1] >= 0)
                                        asm volatile("ld.shared.u16 %0, [%1];" : "=h"(hi) : "r"(xr + (uint32_t)(tv[2 * e + 1] * 2)));
                                    w[e] = (uint32_t)lo | ((uint32_t)hi << 16);
                                }
                            }
                        }
                        asm volatile("st.shared.v4.b32 [%0], {%1, %2, %3, %4};" ::"r"(aT + kmaj_off(i, c8 * 16)),
                                     "r"(w[0]), "r"(w[1]), "r"(w[2]), "r"(w[3])
                                     : "memory");
                    }
                    fence_proxy_async();
                    mbar_arrive(smem_u32(&full[s]));
                }
                mbar_arrive(smem_u32(&xempty[jx]));
            }
        }
    }
    if ((STAGED || STAGED_FWD) && (warp < 4 || warp == 9)) {
        // builders / TMA warp only (above)
    } else if (HALO && warp < 4) {

        // ===================== halo producers (A_HALO) =====================
        // warp 1: one halo per (tile, channel chunk) = the full rows of the
        // extended source grid the tile's taps touch (one TMA row box each);
        // warp 0: the filter k-block of every (tile, chunk, tap).  Whole warps
        // run the loops (lane 0 issues): a lone spinning lane next to lanes
        // parked at the CTA barrier starves (measured 2x slower).
        const int taps = p.tapR * p.tapS;
        if (warp == 1) {
            int hs = 0;
            uint32_t hph = 0;
            for (int tile = blockIdx.x; tile < total_tiles; tile += gridDim.x) {
                int m0, n0, z, kb_begin, kb_end;
                decode(tile, m0, n0, z, kb_begin, kb_end);
                const int G0 = m0 / p.hx_W;
                const int G1 = (m0 + BMt - 1 + (p.tapR - 1) * p.hx_W + p.tapS - 1) / p.hx_W;
                const int nr = G1 - G0 + 1;
                for (int c = 0; c < p.hx_nch; ++c) {
                    mbar_wait(smem_u32(&hempty[hs]), hph ^ 1u);
                    if (lane == 0) {
                        const uint32_t dst = smem_u32(sA + (size_t)hs * p.halo_bytes);
                        const uint32_t fb = smem_u32(&hfull[hs]);
                        mbar_arrive_tx(fb, (uint32_t)(nr * p.hx_W * 128));
                        int n_ = G0 / p.hx_H, hx = G0 - n_ * p.hx_H;
                        for (int i = 0; i < nr; ++i) {
                            tma_load_4d(dst + (uint32_t)(i * p.hx_W * 128), &tmA, fb, c * KB, -p.hx_pe,
                                        hx - p.hx_pe, n_);
                            if (++hx == p.hx_H) { hx = 0; ++n_; }
                        }
                    }
                    __syncwarp();
                    if (++hs == p.hstages) { hs = 0; hph ^= 1u; }
                }
            }
        } else if (warp == 0) {
            int s = 0;
            uint32_t ph = 0;
            for (int tile = blockIdx.x; tile < total_tiles; tile += gridDim.x) {
                int m0, n0, z, kb_begin, kb_end;
                decode(tile, m0, n0, z, kb_begin, kb_end);
                for (int c = 0; c < p.hx_nch; ++c) {
                    for (int tap = 0; tap < taps; ++tap) {
                        mbar_wait(smem_u32(&empty[s]), ph ^ 1u);
                        if (lane == 0) {
                            const uint32_t bT = smem_u32(sB + (size_t)s * B_BYTES);
                            const uint32_t fb = smem_u32(&full[s]);
                            mbar_arrive_tx(fb, (uint32_t)p.tma_bytes);
                            if constexpr (BM_ == B_TMA_K2) tma_load_2d(bT, &tmB, fb, tap * p.C + c * KB, n0);
                            if constexpr (BM_ == B_TMA_MN3) {
                                // DGRAD: tap (r', s') of the flipped filter = w[.][R-1-r'][S-1-s'][.]
                                const int rr = tap / p.tapS, ss = tap - rr * p.tapS;
                                const int rs = (p.R - 1 - rr) * p.S + (p.S - 1 - ss);
                                for (int a = 0; a < p.bn_atoms; ++a)
                                    tma_load_3d(bT + a * KB * 128, &tmB, fb, n0 + a * (128 / ELT), rs, c * KB);
                            }
                        }
                        __syncwarp();
                        if (++s == S) { s = 0; ph ^= 1u; }
                    }
                }
            }
        }
    } else if (warp < 4) {
        // =========================== producers ===========================
        const int t = threadIdx.x;  // 0..127
        const T* gx = (const T*)p.gsrc;
        const int lag = min(S - 1, p.max_lag);
        const int gch = (AM == A_GATHER_DGRAD || (AM == A_TMA_IM2COL && p.im2col_dgrad)) ? p.K : p.C;
        if constexpr (B_RES) {
            // Stage the whole zero-padded filter once: B(n, k') with k' = (r, s8, c')
            // -> w[n][r][s][c'] (0 for s >= S or c' >= C), K-major SW128 per k-block.
            const T* wsrc = (const T*)p.bsrc;
            const int groups = p.s8 / 8;  // tap groups of 8 per filter row
            const int per_kb = p.BN * KB;
            for (int idx = t; idx < p.num_kb * per_kb; idx += 128) {
                const int kb = idx / per_kb, rem = idx - kb * per_kb;
                const int n = rem / KB, e = rem - n * KB;
                const int r = kb / groups, s_ = (kb - r * groups) * 8 + e / p.cp, c = e % p.cp;
                float v = 0.f;
                if (n < p.N && s_ < p.S && c < p.C) v = (float)wsrc[(((size_t)n * p.R + r) * p.S + s_) * p.C + c];
                st_shared_elt<T>(smem_u32(sBres) + (uint32_t)(kb * p.BN * 128) + kmaj_off(n, e * ELT), (T)v);
            }
            fence_proxy_async();
            mbar_arrive(smem_u32(bres_bar));
        }
        int s = 0;
        uint32_t ph = 0;
        int git = 0;  // k-blocks issued by this CTA so far (for the lagged arrivals)
        // TMA-only operands (no gathers): warp 0 runs the stage loop (lane 0 issues) and
        // warps 1-3 stay out of it.  A thread that only waits on the empty barriers
        // without gating them can fall two phases behind (a concurrent kernel delaying
        // its warp): the barrier's parity then repeats and its last wait never returns
        // (observed: a hang at the end of the tile loop under the concurrent backward).
        // (Warp 0's other lanes wait alongside lane 0, which gates every stage it waits
        // for; a __syncwarp per stage to pin them costs 10 % on short ResNet layers.)
        const bool in_loop = GATHER || warp == 0;
        for (int tile = in_loop ? (int)blockIdx.x : total_tiles; tile < total_tiles; tile += gridDim.x) {
            int m0, n0, z, kb_begin, kb_end;
            decode(tile, m0, n0, z, kb_begin, kb_end);
            // Per-thread gather rows (A gathers: rows t/8 + 16 i, chunk t % 8):
            // FWD  row = output pixel (n,p,q): origin (p*st - pad, q*st - pad) in x,
            //      element (r,s,c) at base + (r*W + s)*C + c;
            // DGRAD row = dx pixel (n,h,w): dy index (h + pad - r, w + pad - s)
            //      (stride 1: element (r,s,k) at base - (r*Q + s)*K + k).
            int rh[8], rw[8];
            long long rbase[8];
            bool rv[8];
            if constexpr (AM == A_GATHER_FWD || AM == A_GATHER_DGRAD || AM == A_GATHER_SMALLC ||
                          AM == A_GATHER_SMALLC_PAD) {
#pragma unroll
                for (int i = 0; i < 8; ++i) {
                    const int m = m0 + t / 8 + 16 * i;
                    rv[i] = m < p.M;
                    const int mm = rv[i] ? m : 0;
                    if (AM == A_GATHER_FWD || AM == A_GATHER_SMALLC || AM == A_GATHER_SMALLC_PAD) {
                        const int pq = p.P * p.Q;
                        const int n = mm / pq, rem = mm - n * pq, pp = rem / p.Q, qq = rem - pp * p.Q;
                        rh[i] = pp * p.stride - p.pad; rw[i] = qq * p.stride - p.pad;
                        rbase[i] = (((long long)n * p.H + rh[i]) * p.W + rw[i]) *
                                   (AM == A_GATHER_SMALLC_PAD ? p.cp : p.C);
                    } else {
                        const int hw = p.H * p.W;
                        const int n = mm / hw, rem = mm - n * hw, hh = rem / p.W, ww = rem - hh * p.W;
                        rh[i] = hh + p.pad; rw[i] = ww + p.pad;
                        rbase[i] = p.stride == 1 ? (((long long)n * p.P + rh[i]) * p.Q + rw[i]) * p.K
                                                 : (long long)n * p.P * p.Q * p.K;  // strided: image base
                    }
                }
            }
            // Phase of this tile (merged strided-DGRAD launch: z = phase index)
            int tR = p.tapR, tS = p.tapS, pr0 = p.ph_r0, ps0 = p.ph_s0, pi0 = p.ph_i0, pj0 = p.ph_j0;
            if (p.ph_n) {
                tR = p.ph_tRv[z]; tS = p.ph_tSv[z]; pr0 = p.ph_r0v[z]; ps0 = p.ph_s0v[z];
                pi0 = p.ph_i0v[z]; pj0 = p.ph_j0v[z];
            }
            // Incremental (r, s, c0) of the current k-block: a k-block covers KB
            // consecutive channels of one filter tap.
            int g_c0 = 0, g_s = 0, g_r = 0;
            if constexpr (WALK) {
                const int kk0 = kb_begin * KB;
                const int rs = kk0 / gch;
                g_c0 = kk0 - rs * gch; g_r = rs / tS; g_s = rs - g_r * tS;
            }
            // TMA im2col start pixel of this tile (FWD: output pixel m0 -> x origin;
            // DGRAD: dx pixel m0 -> dy origin h + pad - (R-1); phase mode: sub-grid
            // pixel (ii, jj) -> dy origin (i0 + ii - (tapR-1), j0 + jj - (tapS-1))).
            int ic_w[4] = {0, 0, 0, 0}, ic_h[4] = {0, 0, 0, 0}, ic_n[4] = {0, 0, 0, 0};  // per 128-row block (constant-indexed)
            auto ic_of = [&](int mH, int& icw, int& ich, int& icn) {
                if (p.ph_mode) {
                    const int hw = p.ph_H * p.ph_W;
                    icn = mH / hw;
                    const int rem = mH - icn * hw, ii = rem / p.ph_W, jj = rem - ii * p.ph_W;
                    // ph_u > 1 (space-to-depth DGRAD): the map walks u-strided positions
                    ich = p.ph_u * (pi0 + ii) + (p.ph_u - 1) - (tR - 1);
                    icw = p.ph_u * (pj0 + jj) + (p.ph_u - 1) - (tS - 1);
                } else if (p.im2col_dgrad) {
                    const int hw = p.H * p.W;
                    icn = mH / hw;
                    const int rem = mH - icn * hw, hq = rem / p.W, wq = rem - hq * p.W;
                    ich = hq + p.pad - (p.R - 1); icw = wq + p.pad - (p.S - 1);
                } else {
                    const int pq = p.P * p.Q;
                    icn = mH / pq;
                    const int rem = mH - icn * pq, pp = rem / p.Q, qq = rem - pp * p.Q;
                    ich = pp * p.stride - p.pad; icw = qq * p.stride - p.pad;
                }
            };
            if constexpr (AM == A_TMA_IM2COL) {
#pragma unroll
                for (int hh = 0; hh < 4; ++hh)
                    if (hh < p.mt) ic_of(m0 + 128 * hh, ic_w[hh], ic_h[hh], ic_n[hh]);
            }
            // Small-C FWD gather: packed 16-B chunks of 8 rows for one k-block.
            uint32_t pk[8][4];
            auto smallc_load = [&](int kbl) {
                if constexpr (AM == A_GATHER_SMALLC) {
                    const int groups = p.s8 / 8;
                    const int r = kbl / groups, sx = (kbl - r * groups) * 8 + (t & 7);
                    const long long koff = ((long long)r * p.W + sx) * p.C;
#pragma unroll
                    for (int i = 0; i < 8; ++i) {
                        const bool v = sx < p.S && rv[i] && (unsigned)(rh[i] + r) < (unsigned)p.H &&
                                       (unsigned)(rw[i] + sx) < (unsigned)p.W;
                        __align__(16) T vals[16 / ELT];
#pragma unroll
                        for (int u = 0; u < 16 / ELT; ++u)
                            vals[u] = (v && u < p.C) ? gx[rbase[i] + koff + u] : (T)0.f;
                        const uint4 q = *reinterpret_cast<const uint4*>(vals);
                        pk[i][0] = q.x; pk[i][1] = q.y; pk[i][2] = q.z; pk[i][3] = q.w;
                    }
                }
            };
            // Small-C WGRAD gather: 16-B padded-pixel chunks for KB/16 rows x atoms.
            uint32_t bpk[KB / 16][256 / KB][4];
            auto wg_smallc_load = [&](int kbl) {
                if constexpr (BM_ == B_GATHER_SMALLC) {
                    const int chunk = t & 7;
                    const int groups = p.s8 / 8;
                    const int pq = p.P * p.Q;
#pragma unroll
                    for (int i = 0; i < KB / 16; ++i) {
                        const int m = kbl * KB + t / 8 + 16 * i;
                        const bool mv = m < p.kred;
                        const int mm = mv ? m : 0;
                        const int n = mm / pq, rem = mm - n * pq, pp = rem / p.Q, qq = rem - pp * p.Q;
#pragma unroll
                        for (int a = 0; a < 256 / KB; ++a) {
                            const int grp = (n0 * ELT) / 128 + a;  // tap group index = atom index
                            const int r = grp / groups, sx = (grp - r * groups) * 8 + chunk;
                            const int h = pp * p.stride - p.pad + r, w = qq * p.stride - p.pad + sx;
                            const bool v = a < p.bn_atoms && mv && r < p.R && sx < p.S && h >= 0 && h < p.H &&
                                           w >= 0 && w < p.W;
                            __align__(16) T vals[16 / ELT];
                            const T* src = v ? gx + (((size_t)n * p.H + h) * p.W + w) * p.C : gx;
#pragma unroll
                            for (int u = 0; u < 16 / ELT; ++u) vals[u] = (v && u < p.C) ? src[u] : (T)0.f;
                            const uint4 q = *reinterpret_cast<const uint4*>(vals);
                            bpk[i][a][0] = q.x; bpk[i][a][1] = q.y; bpk[i][a][2] = q.z; bpk[i][a][3] = q.w;
                        }
                    }
                }
            };
            // WGRAD TMA im2col: pixel (n,p,q) of the first row of the k-block,
            // walked incrementally (KB pixels per k-block).
            int wb_n = 0, wb_p = 0, wb_q = 0;
            if constexpr (BM_ == B_TMA_IM2COL) {
                const int m = kb_begin * KD, pq = p.P * p.Q;
                wb_n = m / pq;
                const int rem = m - wb_n * pq;
                wb_p = rem / p.Q; wb_q = rem - wb_p * p.Q;
            }
            // Window WGRAD: k-block kb = (output row n*P + p, q-block qb)
            int wr_row = 0, wr_qb = 0;
            if constexpr (WIN) { wr_row = kb_begin / p.win_qb; wr_qb = kb_begin - wr_row * p.win_qb; }
            for (int kb = kb_begin; kb < kb_end; ++kb, ++git, s = (s + 1 == S) ? 0 : s + 1, ph ^= (s == 0) ? 1u : 0u) {
                mbar_wait(smem_u32(&empty[s]), ph ^ 1u);
                const uint32_t aT = smem_u32(sA + (size_t)s * A_BYTES);
                const uint32_t bT = smem_u32(sB + (size_t)s * B_BYTES);
                const uint32_t fb = smem_u32(&full[s]);
                if ((A_TMA || B_TMA) && t == 0) {
                    mbar_arrive_tx(fb, (uint32_t)p.tma_bytes);
                    // A: p.mt blocks of 128 rows (16 KB each)
#pragma unroll
                    for (int hh = 0; hh < 4; ++hh) {
                        if (hh >= p.mt) break;
                        const uint32_t aH = aT + hh * (A_MN ? (uint32_t)A_HALF : 16384u);
                        const int mH = m0 + 128 * hh;
                        if constexpr (AM == A_TMA_K2) tma_load_2d(aH, &tmA, fb, kb * KB, mH);
                        if constexpr (AM == A_TMA_K3) tma_load_3d(aH, &tmA, fb, kb * KB, mH, z);
                        if constexpr (AM == A_TMA_MN2) {
                            const int zr = p.zsplit ? (z / p.zsplit) * p.zrows : 0;
                            if (p.a_box) {
                                tma_load_3d(aH, &tmA, fb, 0, zr + kb * KD, mH / (128 / ELT));
                            } else {
#pragma unroll
                                for (int a = 0; a < 128 * ELT / 128; ++a)
                                    tma_load_2d(aH + a * KD * 128, &tmA, fb, mH + a * (128 / ELT), zr + kb * KD);
                            }
                        }
                        if constexpr (WIN) {
                            // atom ja = (filter row r, atom aa): window of KD output pixels of row
                            // (n, p) at x row st*p + r - pad (rows past R load out of bounds: zeros);
                            // atoms of aw bytes, 128*ELT/aw of them per 128 rows
                            const int n_ = wr_row / p.P, p_ = wr_row - n_ * p.P;
                            constexpr int wat = WAW / ELT;
                            if (p.win_box) {
                                const int r0 = (mH / wat) / p.win_na;
                                tma_load_5d(aH, &tmA, fb, 0, wr_qb * KD, 0, p.stride * p_ + r0 - p.pad, n_);
                            } else
#pragma unroll
                            for (int a = 0; a < 128 * ELT / (int)WAW; ++a) {
                                const int ja = mH / wat + a;
                                const int r = ja / p.win_na, aa = ja - r * p.win_na;
                                const int h = r < p.R ? p.stride * p_ + r - p.pad : -(1 << 20);
                                tma_load_4d(aH + a * KD * WAW, &tmA, fb, aa * wat, wr_qb * KD, h, n_);
                            }
                        }
                        if constexpr (AM == A_TMA_IM2COL) {
                            // 128 consecutive output pixels x KB channels of tap (r,s) in one TMA
                            // (a_merged: all 128*mt pixels of the tile in the first half's TMA)
                            const uint16_t ow = (uint16_t)(p.im2col_dgrad ? tS - 1 - g_s : g_s);
                            const uint16_t oh = (uint16_t)(p.im2col_dgrad ? tR - 1 - g_r : g_r);
                            if (!p.a_merged || hh == 0)
                                tma_load_im2col_4d(aH, &tmA, fb, g_c0, ic_w[hh], ic_h[hh], ic_n[hh], ow, oh);
                        }
                    }
                    if constexpr (BM_ == B_TMA_K2) tma_load_2d(bT, &tmB, fb, kb * KB, n0);
                    if constexpr (BM_ == B_TMA_K3) tma_load_3d(bT, &tmB, fb, kb * KB, n0, z);
                    if constexpr (BM_ == B_TMA_MN2) {
                        const int zr = p.zsplit ? (z / p.zsplit) * p.zrows : 0;
                        if (p.b_box) {
                            tma_load_3d(bT, &tmB, fb, 0, zr + kb * KD, n0 / (128 / ELT));
                        } else {
                            for (int a = 0; a < p.bn_atoms; ++a)
                                tma_load_2d(bT + a * KD * 128, &tmB, fb, n0 + a * (128 / ELT), zr + kb * KD);
                        }
                    }
                    if constexpr (BM_ == B_TMA_MN3) {
                        // k-block kb covers tap kb / (K/KB), channels k0 = (kb % (K/KB)) * KB
                        const int kpr = p.K / KB;
                        const int tap = kb / kpr, k0 = (kb - tap * kpr) * KB;
                        const int rs = dgrad_tap_rs(p, tap, pr0, ps0, tS);
                        if (p.b_box) {
                            tma_load_4d(bT, &tmB, fb, 0, rs, k0, n0 / (128 / ELT));
                        } else {
                            for (int a = 0; a < p.bn_atoms; ++a)
                                tma_load_3d(bT + a * KB * 128, &tmB, fb, n0 + a * (128 / ELT), rs, k0);
                        }
                    }
                    if constexpr (BM_ == B_TMA_DYROW) {
                        for (int a = 0; a < p.bn_atoms; ++a)
                            tma_load_3d(bT + a * KD * 128, &tmB, fb, n0 + a * (128 / ELT), wr_qb * KD, wr_row);
                    }
                    if constexpr (BM_ == B_TMA_IM2COL) {
                        // atom a = 128 B of channels (c0..) of tap (r,s) for KB pixels
                        const int h0 = wb_p * p.stride - p.pad, w0 = wb_q * p.stride - p.pad;
                        for (int a = 0; a < p.bn_atoms; ++a) {
                            const int j0 = n0 + a * (128 / ELT);
                            const int rs = j0 / p.C, c0 = j0 - rs * p.C;
                            const int r = rs / p.S, sx = rs - r * p.S;
                            tma_load_im2col_4d(bT + a * KD * 128, &tmB, fb, c0, w0, h0, wb_n, (uint16_t)sx,
                                               (uint16_t)r);
                        }
                    }
                }
                if constexpr (WIN) { if (++wr_qb == p.win_qb) { wr_qb = 0; ++wr_row; } }
                if constexpr (BM_ == B_TMA_IM2COL) {
                    wb_q += KD;
                    while (wb_q >= p.Q) { wb_q -= p.Q; if (++wb_p == p.P) { wb_p = 0; ++wb_n; } }
                }
                // ---- A gathers ----
                if constexpr (AM == A_GATHER_FWD) {
                    const int r = g_r, sx = g_s;
                    const bool kin = r < p.R;
                    const long long koff = ((long long)r * p.W + sx) * p.C + g_c0 + (t & 7) * (16 / ELT);
                    const uint32_t soff = kmaj_off(t / 8, (t & 7) * 16);
#pragma unroll
                    for (int i = 0; i < 8; ++i) {
                        const bool v = kin && rv[i] && (unsigned)(rh[i] + r) < (unsigned)p.H &&
                                       (unsigned)(rw[i] + sx) < (unsigned)p.W;
                        cp_async16(aT + soff + i * 2048, v ? gx + rbase[i] + koff : gx, v);
                    }
                } else if constexpr (AM == A_GATHER_DGRAD) {
                    const int r = g_r, sx = g_s;
                    const bool kin = r < p.R;
                    const int kc = g_c0 + (t & 7) * (16 / ELT);
                    const uint32_t soff = kmaj_off(t / 8, (t & 7) * 16);
                    if (p.stride == 1) {
                        const long long koff = kc - ((long long)r * p.Q + sx) * p.K;
#pragma unroll
                        for (int i = 0; i < 8; ++i) {
                            const bool v = kin && rv[i] && (unsigned)(rh[i] - r) < (unsigned)p.P &&
                                           (unsigned)(rw[i] - sx) < (unsigned)p.Q;
                            cp_async16(aT + soff + i * 2048, v ? gx + rbase[i] + koff : gx, v);
                        }
                    } else {
#pragma unroll
                        for (int i = 0; i < 8; ++i) {
                            const int ph_ = rh[i] - r, pw_ = rw[i] - sx;
                            bool v = kin && rv[i] && ph_ >= 0 && pw_ >= 0;
                            int pp = 0, qq = 0;
                            if (v) {
                                pp = ph_ / p.stride; qq = pw_ / p.stride;
                                v = (pp * p.stride == ph_) && (qq * p.stride == pw_) && pp < p.P && qq < p.Q;
                            }
                            const T* src = v ? gx + rbase[i] + ((long long)pp * p.Q + qq) * p.K + kc : gx;
                            cp_async16(aT + soff + i * 2048, src, v);
                        }
                    }
                }
                if constexpr (AM == A_GATHER_SMALLC_PAD) {
                    // k-block = filter row r, taps s0..s0+7; chunk j = tap s0 + j = one
                    // 16-B padded pixel of the channel-padded x (async, lagged arrive).
                    const int groups = p.s8 / 8;
                    const int r = kb / groups, sx = (kb - r * groups) * 8 + (t & 7);
                    const uint32_t soff = kmaj_off(t / 8, (t & 7) * 16);
                    const long long koff = ((long long)r * p.W + sx) * p.cp;
#pragma unroll
                    for (int i = 0; i < 8; ++i) {
                        const bool v = sx < p.S && rv[i] && (unsigned)(rh[i] + r) < (unsigned)p.H &&
                                       (unsigned)(rw[i] + sx) < (unsigned)p.W;
                        cp_async16(aT + soff + i * 2048, v ? gx + rbase[i] + koff : gx, v);
                    }
                }
                if constexpr (AM == A_GATHER_SMALLC) {
                    // k-block = filter row r, taps s0..s0+7; chunk j = tap s0 + j holds the
                    // pixel's C (< 16 B) channels zero-padded to 16 B.  The registers
                    // were filled one k-block ahead (software pipelining of the
                    // synchronous loads): store them, then prefetch the next k-block.
                    const uint32_t soff = kmaj_off(t / 8, (t & 7) * 16);
                    if (kb == kb_begin) smallc_load(kb);
#pragma unroll
                    for (int i = 0; i < 8; ++i)
                        asm volatile("st.shared.v4.b32 [%0], {%1, %2, %3, %4};" ::"r"(aT + soff + i * 2048),
                                     "r"(pk[i][0]), "r"(pk[i][1]), "r"(pk[i][2]), "r"(pk[i][3])
                                     : "memory");
                }
                if constexpr (WALK) {
                    g_c0 += KB;
                    if (g_c0 >= gch) { g_c0 = 0; if (++g_s == tS) { g_s = 0; ++g_r; } }
                }
                if constexpr (AM == A_SCALAR_FWD) {
                    // thread t owns row t; KB elements, kk = (r,s,c) decomposed each
                    const int m = m0 + t;
                    const bool rvalid = m < p.M;
                    const int pq = p.P * p.Q;
                    const int mm = rvalid ? m : 0;
                    const int n = mm / pq, rem = mm - n * pq, pp = rem / p.Q, qq = rem - pp * p.Q;
                    for (int e = 0; e < KB; ++e) {
                        const int kk = kb * KB + e;
                        float v = 0.f;
                        if (rvalid && kk < p.kred) {
                            const int rs = kk / p.C, c = kk - rs * p.C, r = rs / p.S, sx = rs - r * p.S;
                            const int h = pp * p.stride - p.pad + r, w = qq * p.stride - p.pad + sx;
                            if (h >= 0 && h < p.H && w >= 0 && w < p.W)
                                v = (float)gx[(((size_t)n * p.H + h) * p.W + w) * p.C + c];
                        }
                        st_shared_elt<T>(aT + kmaj_off(t, e * ELT), (T)v);
                    }
                } else if constexpr (AM == A_SCALAR_DGRAD) {
                    // thread t owns dx pixel row t; kk = (r,s,k) decomposed per element
                    const int m = m0 + t;
                    const bool rvalid = m < p.M;
                    const int hw = p.H * p.W;
                    const int mm = rvalid ? m : 0;
                    const int n = mm / hw, rem = mm - n * hw, hh = rem / p.W, ww = rem - hh * p.W;
                    for (int e = 0; e < KB; ++e) {
                        const int kk = kb * KB + e;
                        float v = 0.f;
                        if (rvalid && kk < p.kred) {
                            const int rs = kk / p.K, k = kk - rs * p.K, r = rs / p.S, sx = rs - r * p.S;
                            const int ph_ = hh + p.pad - r, pw_ = ww + p.pad - sx;
                            if (ph_ >= 0 && pw_ >= 0 && ph_ % p.stride == 0 && pw_ % p.stride == 0) {
                                const int pp = ph_ / p.stride, qq = pw_ / p.stride;
                                if (pp < p.P && qq < p.Q)
                                    v = (float)gx[(((size_t)n * p.P + pp) * p.Q + qq) * p.K + k];
                            }
                        }
                        st_shared_elt<T>(aT + kmaj_off(t, e * ELT), (T)v);
                    }
                }
                // ---- B gathers ----
                if constexpr (BM_ == B_GATHER_WG) {
                    // KB pixel rows x bn_atoms atoms x 8 chunks; thread: chunk t%8, rows t/8 + 16 i
                    const int chunk = t & 7;
                    for (int i = 0; i < KB / 16; ++i) {
                        const int row = t / 8 + 16 * i;
                        const int m = kb * KB + row;
                        const int pq = p.P * p.Q;
                        const bool mv = m < p.kred;
                        const int mm = mv ? m : 0;
                        const int n = mm / pq, rem = mm - n * pq, pp = rem / p.Q, qq = rem - pp * p.Q;
                        for (int a = 0; a < p.bn_atoms; ++a) {
                            const int j0 = n0 + a * (128 / ELT);
                            const int rs = j0 / p.C, c0 = j0 - rs * p.C + chunk * (16 / ELT);
                            const int r = rs / p.S, sx = rs - r * p.S;
                            const int h = pp * p.stride - p.pad + r, w = qq * p.stride - p.pad + sx;
                            const bool v = mv && rs < p.R * p.S && h >= 0 && h < p.H && w >= 0 && w < p.W;
                            const T* src = v ? gx + (((size_t)n * p.H + h) * p.W + w) * p.C + c0 : gx;
                            cp_async16(bT + (uint32_t)(a * KB * 128) + mn_row_off<ELT>(row, chunk * 16), src, v);
                        }
                    }
                } else if constexpr (BM_ == B_GATHER_SMALLC_PAD) {
                    // WGRAD small C from padded x: atom = tap group (r, s0..s0+7),
                    // chunk = tap, one 16-B cp.async per (pixel row, tap).
                    const int chunk = t & 7;
                    const int groups = p.s8 / 8;
                    const int pq = p.P * p.Q;
                    for (int i = 0; i < KB / 16; ++i) {
                        const int row = t / 8 + 16 * i;
                        const int m = kb * KB + row;
                        const bool mv = m < p.kred;
                        const int mm = mv ? m : 0;
                        const int n = mm / pq, rem = mm - n * pq, pp = rem / p.Q, qq = rem - pp * p.Q;
                        for (int a = 0; a < p.bn_atoms; ++a) {
                            const int grp = (n0 * ELT) / 128 + a;
                            const int r = grp / groups, sx = (grp - r * groups) * 8 + chunk;
                            const int h = pp * p.stride - p.pad + r, w = qq * p.stride - p.pad + sx;
                            const bool v = mv && r < p.R && sx < p.S && h >= 0 && h < p.H && w >= 0 && w < p.W;
                            const T* src = v ? gx + (((size_t)n * p.H + h) * p.W + w) * p.cp : gx;
                            cp_async16(bT + (uint32_t)(a * KB * 128) + mn_row_off<ELT>(row, chunk * 16), src, v);
                        }
                    }
                } else if constexpr (BM_ == B_GATHER_SMALLC) {
                    // WGRAD small C: B(j' = (r, s8, c'), m) MN-major; an atom (128 B)
                    // is one tap group (r, s0..s0+7), chunk = tap, 16 B = padded pixel.
                    // Registers filled one k-block ahead (see wg_smallc_load).
                    const int chunk = t & 7;
                    if (kb == kb_begin) wg_smallc_load(kb);
#pragma unroll
                    for (int i = 0; i < KB / 16; ++i)
#pragma unroll
                        for (int a = 0; a < 256 / KB; ++a)
                            if (a < p.bn_atoms)
                                asm volatile("st.shared.v4.b32 [%0], {%1, %2, %3, %4};" ::"r"(
                                                 bT + (uint32_t)(a * KB * 128) +
                                                 mn_row_off<ELT>(t / 8 + 16 * i, chunk * 16)),
                                             "r"(bpk[i][a][0]), "r"(bpk[i][a][1]), "r"(bpk[i][a][2]),
                                             "r"(bpk[i][a][3])
                                             : "memory");
                } else if constexpr (BM_ == B_SCALAR_K) {
                    // B rows n0.. (BN of them) x KB elements from a dense row-major matrix with pitch ldb
                    const T* bs = (const T*)p.bsrc;
                    for (int idx = t; idx < p.BN * KB; idx += 128) {
                        const int row = idx / KB, e = idx - (idx / KB) * KB;
                        const int j = n0 + row, kk = kb * KB + e;
                        const float v = (j < p.N && kk < p.kred) ? (float)bs[(size_t)j * p.ldb + kk] : 0.f;
                        st_shared_elt<T>(bT + kmaj_off(row, e * ELT), (T)v);
                    }
                } else if constexpr (BM_ == B_SCALAR_DGRAD) {
                    // B(j = c, kk = (r,s,k)) = w[k][r][s][c], MN-major
                    const T* bs = (const T*)p.bsrc;
                    const int RS = p.R * p.S;
                    for (int idx = t; idx < p.BN * KB; idx += 128) {
                        const int krow = idx / p.BN, jj = idx - krow * p.BN;
                        const int j = n0 + jj, kk = kb * KB + krow;
                        float v = 0.f;
                        if (j < p.N && kk < p.kred) {
                            const int tap = kk / p.K, k = kk - tap * p.K;
                            const int rs = dgrad_tap_rs(p, tap, pr0, ps0, tS);
                            v = (float)bs[((size_t)k * RS + rs) * p.C + j];
                        }
                        st_shared_elt<T>(bT + mnmaj_off<ELT>(jj, krow, KB), (T)v);
                    }
                } else if constexpr (BM_ == B_SCALAR_WG) {
                    // B(j = (r,s,c), kk = pixel m) = x[n, p*st + r - pad, q*st + s - pad, c], MN-major
                    const int pq = p.P * p.Q;
                    for (int idx = t; idx < p.BN * KB; idx += 128) {
                        const int krow = idx / p.BN, jj = idx - krow * p.BN;
                        const int j = n0 + jj, m = kb * KB + krow;
                        float v = 0.f;
                        if (j < p.N && m < p.kred) {
                            const int n = m / pq, rem = m - n * pq, pp = rem / p.Q, qq = rem - pp * p.Q;
                            const int rs = j / p.C, c = j - rs * p.C, r = rs / p.S, sx = rs - r * p.S;
                            const int h = pp * p.stride - p.pad + r, w = qq * p.stride - p.pad + sx;
                            if (h >= 0 && h < p.H && w >= 0 && w < p.W)
                                v = (float)gx[(((size_t)n * p.H + h) * p.W + w) * p.C + c];
                        }
                        st_shared_elt<T>(bT + mnmaj_off<ELT>(jj, krow, KB), (T)v);
                    }
                }
                if constexpr (GATHER) {
                    if constexpr (A_ASYNC || B_ASYNC) {
                        cp_async_commit();
                        // Lagged arrive: keep `lag` stages of gathers in flight per
                        // thread (L2 latency hiding); stage git-lag is complete once
                        // at most `lag` groups are pending.  lag <= S-1 keeps the
                        // ring deadlock-free (the MMA can always drain stage git-S).
                        if (git >= lag) {
                            if (lag == 1) cp_async_wait<1>();
                            else if (lag == 2) cp_async_wait<2>();
                            else if (lag == 3) cp_async_wait<3>();
                            else if (lag == 4) cp_async_wait<4>();
                            else if (lag == 5) cp_async_wait<5>();
                            else cp_async_wait<6>();
                            fence_proxy_async();
                            mbar_arrive(smem_u32(&full[s - lag < 0 ? s - lag + S : s - lag]));
                        }
                    } else {
                        fence_proxy_async();
                        mbar_arrive(fb);
                    }
                }
                // Small-C gathers: prefetch the next k-block's pixels into registers
                // after this stage is published (a fence would otherwise wait for them).
                if constexpr (AM == A_GATHER_SMALLC) { if (kb + 1 < kb_end) smallc_load(kb + 1); }
                if constexpr (BM_ == B_GATHER_SMALLC) { if (kb + 1 < kb_end) wg_smallc_load(kb + 1); }
            }
        }
        if constexpr (GATHER && (A_ASYNC || B_ASYNC)) {
            cp_async_wait<0>();
            fence_proxy_async();
            for (int j = 1; j <= min(lag, git); ++j) mbar_arrive(smem_u32(&full[s - j < 0 ? s - j + S : s - j]));
        }
    } else if (warp == 4) {
        // ======================= MMA issuer (warp 4) =======================
        const uint32_t idesc = (1u << 4) | (Elt<ELT>::fmt << 7) | (Elt<ELT>::fmt << 10) |
                               ((A_MN ? 1u : 0u) << 15) | ((B_MN ? 1u : 0u) << 16) |
                               ((uint32_t)(p.BN >> 3) << 17) | ((128u >> 4) << 24);
        // p.m64: the last 128-row half of the tile holds <= 64 valid rows -> M = 64 MMAs
        // (half the A operand reads; accumulator rows in TMEM lanes 0-15 of each quadrant)
        const uint32_t idesc64 = (idesc & ~(0x1Fu << 24)) | ((64u >> 4) << 24);
        int s = 0;
        uint32_t ph = 0;
        int acc = 0;
        uint32_t aph = 0;
        const int KDm = A_MN ? KD : KB;  // K rows per MN-major atom column (km > 1 only with A_MN)
        if constexpr (B_RES) mbar_wait(smem_u32(bres_bar), 0u);  // staged filter is ready
        if constexpr (HALO) {
            // A for tap (r', s') = 128 consecutive rows of the halo starting at row
            // (m0 - G0*W') + r'*W' + s' -- a shifted window of the same smem tile
            // (SW128 swizzle is address-based, so any 128-B row offset is a valid start).
            int hs = 0;
            uint32_t hph = 0;
            const int taps = p.tapR * p.tapS;
            for (int tile = blockIdx.x; tile < total_tiles; tile += gridDim.x) {
                int m0, n0, z, kb_begin, kb_end;
                decode(tile, m0, n0, z, kb_begin, kb_end);
                mbar_wait(smem_u32(&tempty[acc]), aph ^ 1u);
                tc_fence_after();
                const uint32_t dtm = tmem + (uint32_t)(acc * p.mt * p.BN);
                const int off0 = m0 - (m0 / p.hx_W) * p.hx_W;
                for (int c = 0; c < p.hx_nch; ++c) {
                    mbar_wait(smem_u32(&hfull[hs]), hph);
                    const uint32_t hbase = smem_u32(sA + (size_t)hs * p.halo_bytes) + (uint32_t)(off0 * 128);
                    for (int tap = 0; tap < taps; ++tap) {
                        mbar_wait(smem_u32(&full[s]), ph);
                        tc_fence_after();
                        if (lane == 0) {
                            const int rr = tap / p.tapS;
                            const int ss = tap - rr * p.tapS;
                            const uint32_t aT = hbase + (uint32_t)((rr * p.hx_W + ss) * 128);
                            const uint32_t bT = smem_u32(sB + (size_t)s * B_BYTES);
#pragma unroll
                            for (int j = 0; j < KB / UMMA_K; ++j) {
                                const uint64_t bd = B_MN ? sdesc(bT + j * UMMA_K * 128, KB * 128, MN_SBO, MN_LAYOUT)
                                                         : sdesc(bT + j * 32, 16, 1024);
                                const uint32_t accf = (c > 0 || tap > 0 || j > 0) ? 1u : 0u;
                                mma<ELT>(dtm, sdesc(aT + j * 32, 16, 1024), bd, idesc, accf);
                                if (p.mt == 2)
                                    mma<ELT>(dtm + (uint32_t)p.BN, sdesc(aT + 128 * 128 + j * 32, 16, 1024), bd, idesc,
                                             accf);
                            }
                            mma_commit(smem_u32(&empty[s]));
                            if (tap == taps - 1) mma_commit(smem_u32(&hempty[hs]));
                        }
                        __syncwarp();
                        if (++s == S) { s = 0; ph ^= 1u; }
                    }
                    if (++hs == p.hstages) { hs = 0; hph ^= 1u; }
                }
                if (lane == 0) mma_commit(smem_u32(&tfull[acc]));
                __syncwarp();
                if (++acc == p.nacc) { acc = 0; aph ^= 1u; }
            }
        }
        for (int tile = blockIdx.x; tile < total_tiles && !HALO; tile += gridDim.x) {
            int m0, n0, z, kb_begin, kb_end;
            decode(tile, m0, n0, z, kb_begin, kb_end);
            mbar_wait(smem_u32(&tempty[acc]), aph ^ 1u);  // epilogue has drained this accumulator
            tc_fence_after();
            const uint32_t dtm = tmem + (uint32_t)(acc * p.mt * p.BN);
            int sqb = STAGED ? kb_begin % p.win_qb : 0;  // A_STAGED_WG: q-block of kb (incremental)
            for (int kb = kb_begin; kb < kb_end; ++kb, s = (s + 1 == S) ? 0 : s + 1, ph ^= (s == 0) ? 1u : 0u) {
                mbar_wait(smem_u32(&full[s]), ph);
                tc_fence_after();
                // whole warp (converged): elect.sync inside the MMA / commit picks the issuer
                {
                    const uint32_t aT = smem_u32(sA + (size_t)s * A_BYTES);
                    const uint32_t bT = B_RES ? smem_u32(sBres) + (uint32_t)(kb * p.BN * 128)
                                              : smem_u32(sB + (size_t)s * B_BYTES);
                    // p.mt independent accumulators (one per 128-row half) share B and
                    // interleave, so short-N MMAs are not serialised on one accumulator.
                    // Fully unrolled with compile-time strides: the single issuing thread
                    // is on the critical path (measured: runtime strides / extra variants
                    // here cost 10-30% on the FWD kernels).
                    // A_STAGED_WG: the last pixel block of an output row issues only the MMA K
                    // steps that cover its valid pixels
                    int jmax = KB / UMMA_K;
                    if constexpr (STAGED) {
                        jmax = min(jmax, (min(KD, p.Q - sqb * KD) + UMMA_K - 1) / UMMA_K);
                        if (++sqb == p.win_qb) sqb = 0;
                    }
                    auto issue = [&](auto mt_c, const int jj) {
                        constexpr int MT = decltype(mt_c)::value;
                        // MN-major operands: k-block jj of the stage starts jj * KB rows in
                        const uint32_t kofs = A_MN ? (uint32_t)(jj * KB * 128) : 0u;
#pragma unroll
                        for (int j = 0; j < KB / UMMA_K; ++j) {
                            if (STAGED && j >= jmax) break;
                            const uint64_t bd = B_MN ? sdesc(bT + kofs + j * UMMA_K * 128, KDm * 128, MN_SBO, MN_LAYOUT)
                                                     : sdesc(bT + j * 32, 16, 1024);
#pragma unroll
                            for (int hh = 0; hh < MT; ++hh) {
                                const uint32_t aH = aT + hh * (A_MN ? (uint32_t)A_HALF : 16384u);
                                // window atoms of aw bytes: KD rows x aw per atom column, 8-row
                                // groups aw*8 apart; UMMA swizzle 2 / 4 / 6 = 128 / 64 / 32 B
                                const uint64_t ad =
                                    WIN && WAW < 128
                                        ? sdesc(aH + (uint32_t)(jj * KB) * WAW + j * UMMA_K * WAW, KDm * WAW, 8 * WAW,
                                                WAW == 64 ? 4u : 6u)
                                    : A_MN  ? sdesc(aH + kofs + j * UMMA_K * 128, KDm * 128, MN_SBO, MN_LAYOUT)
                                            : sdesc(aH + j * 32, 16, 1024);
                                mma_elect<ELT>(dtm + (uint32_t)(hh * p.BN), ad, bd,
                                               (A_MN && hh == MT - 1 && p.m64) ? idesc64 : idesc,
                                               (kb > kb_begin || jj > 0 || j > 0) ? 1u : 0u);
                            }
                        }
                    };
                    if constexpr (A_MN) {
                        for (int jj = 0; jj < p.km; ++jj) {
                            if (p.mt == 4) issue(std::integral_constant<int, 4>{}, jj);
                            else if (p.mt == 3 && STAGED) issue(std::integral_constant<int, 3>{}, jj);
                            else if (p.mt == 2) issue(std::integral_constant<int, 2>{}, jj);
                            else issue(std::integral_constant<int, 1>{}, jj);
                        }
                    } else {
                        if (p.mt == 4) issue(std::integral_constant<int, 4>{}, 0);
                        else if (p.mt == 2) issue(std::integral_constant<int, 2>{}, 0);
                        else issue(std::integral_constant<int, 1>{}, 0);
                    }
                    mma_commit_elect(smem_u32(&empty[s]));
                }
                __syncwarp();
            }
            if (lane == 0) {
                if (kb_end > kb_begin) mma_commit(smem_u32(&tfull[acc]));
                else mbar_arrive(smem_u32(&tfull[acc]));
            }
            __syncwarp();
            if (++acc == p.nacc) { acc = 0; aph ^= 1u; }
        }
    } else {
        // ============================ epilogue =============================
        const int q4 = warp & 3;  // TMEM lane quadrant of this warp
        const int row = q4 * 32 + lane;
        int acc = 0;
        uint32_t aph = 0;
        if (SPLITK && p.cl) {
            // Cluster split-K: stage alpha * partial (fp32) over the operand ring, row-major
            // with a pitch of BN + 4 floats; the cluster reduces it after the barrier below.
            int m0, n0, z, kb_begin, kb_end;
            decode(blockIdx.x, m0, n0, z, kb_begin, kb_end);
            mbar_wait(smem_u32(&tfull[0]), 0u);
            tc_fence_after();
            const uint32_t stg = smem_u32(smem);
            const int pitch = p.BN + 4;
            for (int hh = 0; hh < p.mt; ++hh) {
                for (int c0 = 0; c0 < p.BN; c0 += 32) {
                    uint32_t v[32];
                    if (kb_end > kb_begin) {
                        TMEM_LD32(tmem + (uint32_t)(hh * p.BN + c0) + ((uint32_t)(q4 * 32) << 16), v);
                        asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
                    } else {
#pragma unroll
                        for (int j = 0; j < 32; ++j) v[j] = 0u;
                    }
                    const bool h64 = p.m64 && hh == p.mt - 1;  // M = 64 half: rows 16*q4 + lane (lane < 16)
                    if (h64 && lane >= 16) continue;
                    const int srow = h64 ? 16 * q4 + lane : row;
                    const uint32_t dst = stg + (uint32_t)(((hh * 128 + srow) * pitch + c0) * 4);
#pragma unroll
                    for (int j = 0; j < 32; j += 4)
                        asm volatile("st.shared.v4.f32 [%0], {%1, %2, %3, %4};" ::"r"(dst + j * 4),
                                     "f"(p.alpha * __uint_as_float(v[j])), "f"(p.alpha * __uint_as_float(v[j + 1])),
                                     "f"(p.alpha * __uint_as_float(v[j + 2])), "f"(p.alpha * __uint_as_float(v[j + 3]))
                                     : "memory");
                }
            }
            tc_fence_before();
        }
        for (int tile = blockIdx.x; tile < total_tiles && !(SPLITK && p.cl); tile += gridDim.x) {
            int m0, n0, z, kb_begin, kb_end;
            decode(tile, m0, n0, z, kb_begin, kb_end);
            const bool has_acc = kb_end > kb_begin;
            mbar_wait(smem_u32(&tfull[acc]), aph);
            tc_fence_after();
            // BackwardFilter without a split (the whole reduction in this CTA):
            // dw = alpha * acc + beta * dw.  Deterministic split reductions take the
            // cluster path; p.atomic (non-deterministic mode) adds every split's partial
            // with L2 reductions after a beta prescale launch.
            const float bsplit = p.beta;
            // NEXT-3: the cross-rank sum target (the final values: no split here) and the
            // element offset of a dw pointer
            const RedTarget* redp = p.red.n ? &p.red : nullptr;
            auto roff = [&](const float* d) -> long long { return (long long)(d - (const float*)p.out); };
            auto drain = [&](const int hh) {
            // M = 64 half: TMEM lane 32*q4 + l (l < 16) holds row 16*q4 + l
            const bool h64 = p.m64 && hh == p.mt - 1;
            const int m = h64 ? (lane < 16 ? m0 + 128 * hh + 16 * q4 + lane : INT_MAX) : m0 + 128 * hh + row;
            // Output row of GEMM row m (phase mode scatters sub-grid rows back to dx).
            long long mrow = m;
            bool rowok = true;
            if (STAGED_FWD && m < p.M) {
                // tile = win_qb output rows of one image: row i = t*Q + q of the tile
                const int tile = m >> 7, i = m & 127, Tr = p.win_qb;
                const int tiles_img = (p.P + Tr - 1) / Tr;
                const int n = tile / tiles_img, pr = (tile - n * tiles_img) * Tr + i / p.Q, q = i % p.Q;
                rowok = i < Tr * p.Q && pr < p.P;
                mrow = ((long long)n * p.P + pr) * p.Q + q;
            }
            if (HALO && m < p.M) {
                // extended-grid row m = ((n*Hx + oh)*W' + ow): junk unless oh < Ho, ow < Wo
                const int G = m / p.hx_W, ow = m - G * p.hx_W, n = G / p.hx_H, oh = G - n * p.hx_H;
                rowok = oh < p.hx_Ho && ow < p.hx_Wo;
                mrow = ((long long)n * p.hx_Ho + oh) * p.hx_Wo + ow;
            }
            if (EPI == EPI_STORE && p.ph_mode && m < p.M) {
                const int hw = p.ph_H * p.ph_W;
                const int n = m / hw, rem = m - n * hw, ii = rem / p.ph_W, jj = rem - ii * p.ph_W;
                const int hb = p.ph_n ? p.ph_hbv[z] : p.ph_hb, wb = p.ph_n ? p.ph_wbv[z] : p.ph_wb;
                mrow = ((long long)n * p.H + hb + p.stride * ii) * p.W + wb + p.stride * jj;
            }
            const uint32_t taddr_row =
                tmem + (uint32_t)((acc * p.mt + hh) * p.BN) + ((uint32_t)(q4 * 32) << 16);
            float* outF = (float*)p.out;
            T* outT = (T*)p.out;
            if (EPI == EPI_STORE && z > 0 && !p.ph_n) {
                outF += (size_t)z * p.batch_stride;
                outT += (size_t)z * p.batch_stride;
            }
            if constexpr (EPI == EPI_D2S) {
                if (p.d2s_rows) {
                    // Depth-to-space by dx rows (beta = 0, one N tile): for each row a of
                    // the f x f super-pixel, its f*C contiguous dx values are read from
                    // TMEM in 4-column pieces (warp-uniform loop: tcgen05.ld is
                    // .sync.aligned) and stored as bf16x2 / float2 words when the segment
                    // lies inside the image (~1.5 instructions per element instead of ~15
                    // with per-column index stepping, which made this epilogue the bound
                    // of the space-to-depth DGRAD); edge super-pixels go element-wise.
                    const bool mv = m < p.M && rowok;
                    const int hw = p.ph_H * p.ph_W;
                    const int mm = mv ? m : 0;
                    const int n = mm / hw, rem = mm - n * hw, ii = rem / p.ph_W, jj = rem - ii * p.ph_W;
                    const int f = p.s2_st, C = p.e_C, fC = f * C;
                    const int h0 = f * ii - p.e_pad, w0 = f * jj - p.e_pad;
                    const bool inner = w0 >= 0 && w0 + f <= p.e_W;
                    const uint32_t tb = tmem + (uint32_t)((acc * p.mt + hh) * p.BN) + ((uint32_t)(q4 * 32) << 16);
                    for (int a = 0; a < f; ++a) {
                        const int h = h0 + a;
                        const bool hv = mv && (unsigned)h < (unsigned)p.e_H;
                        const long long off = (((long long)n * p.e_H + h) * p.e_W + w0) * C;
                        int ebq = 0, ec = 0;  // edge path: (pixel, channel) of element e0 (no division)
                        for (int e0 = 0; e0 < fC; e0 += 4) {
                            uint32_t v[4];
                            if (has_acc) {
                                asm volatile("tcgen05.ld.sync.aligned.32x32b.x4.b32 {%0,%1,%2,%3}, [%4];"
                                             : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3])
                                             : "r"(tb + (uint32_t)(a * fC + e0)));
                                asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
                            } else {
                                v[0] = v[1] = v[2] = v[3] = 0u;
                            }
                            if (!hv) continue;
                            float o[4];
#pragma unroll
                            for (int u = 0; u < 4; ++u) o[u] = p.alpha * __uint_as_float(v[u]);
                            if (inner) {
                                if (p.out_bf16) {
                                    __nv_bfloat16* d = (__nv_bfloat16*)p.out + off + e0;
                                    if ((((uintptr_t)d) & 3) == 0) {
                                        *reinterpret_cast<__nv_bfloat162*>(d) = __floats2bfloat162_rn(o[0], o[1]);
                                        *reinterpret_cast<__nv_bfloat162*>(d + 2) = __floats2bfloat162_rn(o[2], o[3]);
                                    } else {
#pragma unroll
                                        for (int u = 0; u < 4; ++u) d[u] = __float2bfloat16_rn(o[u]);
                                    }
                                } else {
                                    float* d = (float*)p.out + off + e0;
                                    if ((((uintptr_t)d) & 7) == 0) {
                                        *reinterpret_cast<float2*>(d) = make_float2(o[0], o[1]);
                                        *reinterpret_cast<float2*>(d + 2) = make_float2(o[2], o[3]);
                                    } else {
#pragma unroll
                                        for (int u = 0; u < 4; ++u) d[u] = o[u];
                                    }
                                }
                            } else {
#pragma unroll
                                for (int u = 0; u < 4; ++u) {
                                    const int e = e0 + u;
                                    if ((unsigned)(w0 + ebq) < (unsigned)p.e_W) {
                                        if (p.out_bf16) ((__nv_bfloat16*)p.out)[off + e] = __float2bfloat16_rn(o[u]);
                                        else ((float*)p.out)[off + e] = o[u];
                                    }
                                    if (++ec == C) { ec = 0; ++ebq; }
                                }
                            }
                        }
                    }
                    return;
                }
            }
            // EPI_D2S: the row's super-pixel (n, i, j) once per row, not per 32-column chunk
            int d2_n = 0, d2_h0 = 0, d2_w0 = 0;
            if constexpr (EPI == EPI_D2S) {
                if (m < p.M) {
                    const int hw = p.ph_H * p.ph_W;
                    d2_n = m / hw;
                    const int rem = m - d2_n * hw, ii = rem / p.ph_W, jj = rem - ii * p.ph_W;
                    d2_h0 = p.s2_st * ii - p.e_pad;
                    d2_w0 = p.s2_st * jj - p.e_pad;
                }
            }
            for (int c0 = 0; c0 < p.BN; c0 += 32) {
                uint32_t v[32];
                if (has_acc) {
                    TMEM_LD32(taddr_row + (uint32_t)c0, v);
                    asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
                } else {
#pragma unroll
                    for (int j = 0; j < 32; ++j) v[j] = 0u;
                }
                if (m >= p.M || !rowok) continue;
                const int nb = n0 + c0;
                if constexpr (EPI == EPI_D2S) {
                    // super-pixel row (n, i, jj); column (a, b, c) walked incrementally:
                    // the dx offset advances by 1 inside an (a) block of st*C values and
                    // by (W - st)*C between blocks (no per-column index arithmetic).
                    const int n = d2_n, h0 = d2_h0, w0 = d2_w0;
                    const int stc = p.s2_st * p.e_C;
                    int a = nb / stc, bq = (nb - a * stc) / p.e_C, c = nb - a * stc - bq * p.e_C;
                    long long off = (((long long)n * p.e_H + h0 + a) * p.e_W + w0 + bq) * p.e_C + c;
                    const long long jump = (long long)(p.e_W - p.s2_st) * p.e_C;
                    bool okh = (unsigned)(h0 + a) < (unsigned)p.e_H, okw = (unsigned)(w0 + bq) < (unsigned)p.e_W;
                    const int nlim = p.N - nb;
                    if (p.e_C % 32 == 0 && p.beta == 0.f && (((uintptr_t)p.out & 31) == 0)) {
                        // the 32 columns are 32 consecutive channels of one output pixel
                        // (u x u FWD super-pixels): 16-B vector stores
                        if (nlim >= 32 && okh && okw) {
                            if (p.out_bf16) {
                                __nv_bfloat16* d = (__nv_bfloat16*)p.out + off;
#pragma unroll
                                for (int j = 0; j < 32; j += 16) st256_bf16(d + j, v + j, p.alpha);
                            } else {
                                float* d = (float*)p.out + off;
#pragma unroll
                                for (int j = 0; j < 32; j += 8) st256_f32(d + j, v + j, p.alpha);
                            }
                        }
                        continue;
                    }
#pragma unroll
                    for (int j = 0; j < 32; ++j) {
                        if (j < nlim && okh && okw) {
                            float o = p.alpha * __uint_as_float(v[j]);
                            if (p.out_bf16) {
                                __nv_bfloat16* d = (__nv_bfloat16*)p.out + off;
                                if (p.beta != 0.f) o += p.beta * __bfloat162float(*d);
                                *d = __float2bfloat16_rn(o);
                            } else {
                                float* d = (float*)p.out + off;
                                if (p.beta != 0.f) o += p.beta * *d;
                                *d = o;
                            }
                        }
                        ++off;
                        if (++c == p.e_C) {
                            c = 0;
                            if (++bq == p.s2_st) {
                                bq = 0; ++a; off += jump;
                                okh = (unsigned)(h0 + a) < (unsigned)p.e_H;
                            }
                            okw = (unsigned)(w0 + bq) < (unsigned)p.e_W;
                        }
                    }
                } else if constexpr (EPI == EPI_WGRAD_S2D) {
                    // column (tap (d,e), channel (a, b, c)) -> dw[k][st*d+a][st*e+b][c]
                    float* drow = outF + (size_t)m * p.ldc;
                    const int stc = p.s2_st * p.s2_C, real = stc * p.s2_st;
                    int tap = nb / p.C, ch = nb - tap * p.C;
                    int dofs[32];
#pragma unroll
                    for (int j = 0; j < 32; ++j) {
                        dofs[j] = -1;
                        if (nb + j < p.N && ch < real) {
                            const int d = tap / p.S, e = tap - d * p.S;
                            const int a = ch / stc, rem = ch - a * stc, bq = rem / p.s2_C, c = rem - bq * p.s2_C;
                            const int r = p.s2_st * d + a, sx = p.s2_st * e + bq;
                            if (r < p.s2_R && sx < p.s2_S) dofs[j] = (r * p.s2_S + sx) * p.s2_C + c;
                        }
                        if (++ch == p.C) { ch = 0; ++tap; }
                    }
                    rmw32(drow, dofs, 1, v, p.alpha, bsplit, p.atomic, redp, roff(drow));
                } else if constexpr (EPI == EPI_WGRAD_WIN) {
                    // row m = (r, atom aa, tap t, channel c) -> dw[k][r][aa*taps + t][c], k = nb + j
                    constexpr int per_atom = WAW / ELT;
                    const int ja = m / per_atom, e = m - ja * per_atom;
                    const int t = e / p.cp, c = e - t * p.cp;
                    const int r = ja / p.win_na, sx = (ja - r * p.win_na) * (per_atom / p.cp) + t;
                    if (r < p.R && sx < p.S && c < p.C) {
                        float* d = outF + (size_t)nb * p.ldc + (r * p.S + sx) * p.C + c;
                        int dofs[32];
#pragma unroll
                        for (int j = 0; j < 32; ++j) dofs[j] = nb + j < p.N ? j : -1;
                        rmw32(d, dofs, (size_t)p.ldc, v, p.alpha, bsplit, p.atomic, redp, roff(d));
                    }
                } else if constexpr (EPI == EPI_WGRAD_PARTIAL) {
                    // the split's partial tile: out[z][m][nb + j] (rows < part_rows, plain stores)
                    float* d = outF + (size_t)z * p.part_rows * p.ldc + (size_t)m * p.ldc + nb;
                    if (m >= p.part_rows) {
                    } else if (nb + 32 <= p.N && (p.ldc & 3) == 0) {
#pragma unroll
                        for (int j = 0; j < 32; j += 4)
                            *reinterpret_cast<float4*>(d + j) =
                                make_float4(p.alpha * __uint_as_float(v[j]), p.alpha * __uint_as_float(v[j + 1]),
                                            p.alpha * __uint_as_float(v[j + 2]), p.alpha * __uint_as_float(v[j + 3]));
                    } else {
#pragma unroll
                        for (int j = 0; j < 32; ++j)
                            if (nb + j < p.N) d[j] = p.alpha * __uint_as_float(v[j]);
                    }
                } else if constexpr (EPI == EPI_WGRAD_TAPS) {
                    // row m = exact tap (r, s, c) -> dw[k = nb + j][m]
                    if (m < p.kred_taps) {
                        int dofs[32];
#pragma unroll
                        for (int j = 0; j < 32; ++j) dofs[j] = nb + j < p.N ? j : -1;
                        rmw32(outF + (size_t)nb * p.ldc + m, dofs, (size_t)p.ldc, v, p.alpha, bsplit, p.atomic,
                              redp, roff(outF + (size_t)nb * p.ldc + m));
                    }
                } else if constexpr (EPI == EPI_WGRAD_SMALLC) {
                    // padded column j' = (r, s8, c') -> dw column (r*S + s)*C + c (skip padding)
                    float* drow = outF + (size_t)m * p.ldc;
                    int dofs[32];
#pragma unroll
                    for (int j = 0; j < 32; ++j) {
                        const int jp = nb + j;
                        const int c = jp % p.cp, t2 = jp / p.cp, s_ = t2 % p.s8, r = t2 / p.s8;
                        dofs[j] = (jp < p.N && c < p.C && s_ < p.S) ? (r * p.S + s_) * p.C + c : -1;
                    }
                    rmw32(drow, dofs, 1, v, p.alpha, bsplit, p.atomic, redp, roff(drow));
                } else if constexpr (EPI == EPI_WGRAD_CHAIN) {
                    // dw = alpha * partial + bsplit * dw (bsplit = beta on split 0, else 1),
                    // in split order: 16-byte vector read-modify-write
                    float* d = outF + (p.zsplit ? (size_t)(z / p.zsplit) * p.batch_stride : 0) + (size_t)m * p.ldc + nb;
                    const bool vec = (nb + 32 <= p.N) && ((p.ldc & 3) == 0) && ((((uintptr_t)p.out) & 15) == 0);
                    if (vec && p.atomic) {
#pragma unroll
                        for (int j = 0; j < 32; j += 4)
                            asm volatile("red.global.add.v4.f32 [%0], {%1, %2, %3, %4};" ::"l"(d + j),
                                         "f"(p.alpha * __uint_as_float(v[j])), "f"(p.alpha * __uint_as_float(v[j + 1])),
                                         "f"(p.alpha * __uint_as_float(v[j + 2])),
                                         "f"(p.alpha * __uint_as_float(v[j + 3]))
                                         : "memory");
                    } else if (vec) {
                        float4 o[8];
#pragma unroll
                        for (int j = 0; j < 8; ++j)
                            o[j] = bsplit != 0.f ? __ldcg(reinterpret_cast<const float4*>(d) + j)
                                                 : make_float4(0.f, 0.f, 0.f, 0.f);
#pragma unroll
                        for (int j = 0; j < 8; ++j) {
                            float4 q;
                            q.x = p.alpha * __uint_as_float(v[4 * j]) + bsplit * o[j].x;
                            q.y = p.alpha * __uint_as_float(v[4 * j + 1]) + bsplit * o[j].y;
                            q.z = p.alpha * __uint_as_float(v[4 * j + 2]) + bsplit * o[j].z;
                            q.w = p.alpha * __uint_as_float(v[4 * j + 3]) + bsplit * o[j].w;
                            reinterpret_cast<float4*>(d)[j] = q;
                            if (redp) red_add4(p.red, roff(d) + 4 * j, q);
                        }
                    } else {
                        int dofs[32];
#pragma unroll
                        for (int j = 0; j < 32; ++j) dofs[j] = nb + j < p.N ? j : -1;
                        rmw32(d, dofs, 1, v, p.alpha, bsplit, p.atomic, redp, roff(d));
                    }
                } else if (p.out_bf16) {
                    __nv_bfloat16* d = (__nv_bfloat16*)outT + (size_t)mrow * p.ldc + nb;
                    const bool vec = (nb + 32 <= p.N) && ((p.ldc & 7) == 0) && p.beta == 0.f;
                    if (vec && (p.ldc & 15) == 0 && (((uintptr_t)p.out & 31) == 0)) {
                        // 32-B stores: every store fills whole L2 sectors (16-B stores of
                        // rows 512 B apart half-fill them: 2x the L2 write traffic, measured)
#pragma unroll
                        for (int j = 0; j < 32; j += 16) st256_bf16(d + j, v + j, p.alpha);
                    } else if (vec) {
#pragma unroll
                        for (int j = 0; j < 32; j += 8) {
                            __align__(16) __nv_bfloat16 tmp[8];
#pragma unroll
                            for (int u = 0; u < 8; ++u)
                                tmp[u] = __float2bfloat16_rn(p.alpha * __uint_as_float(v[j + u]));
                            *reinterpret_cast<uint4*>(d + j) = *reinterpret_cast<uint4*>(tmp);
                        }
                    } else {
#pragma unroll
                        for (int j = 0; j < 32; ++j) {
                            if (nb + j < p.N) {
                                float o = p.alpha * __uint_as_float(v[j]);
                                if (p.beta != 0.f) o += p.beta * __bfloat162float(d[j]);
                                d[j] = __float2bfloat16_rn(o);
                            }
                        }
                    }
                } else {
                    float* d = outF + (size_t)mrow * p.ldc + nb;
                    const bool vec = (nb + 32 <= p.N) && ((p.ldc & 3) == 0) && p.beta == 0.f;
                    if (vec && (p.ldc & 7) == 0 && (((uintptr_t)p.out & 31) == 0)) {
#pragma unroll
                        for (int j = 0; j < 32; j += 8) st256_f32(d + j, v + j, p.alpha);
                    } else if (vec) {
#pragma unroll
                        for (int j = 0; j < 32; j += 4)
                            *reinterpret_cast<float4*>(d + j) =
                                make_float4(p.alpha * __uint_as_float(v[j]), p.alpha * __uint_as_float(v[j + 1]),
                                            p.alpha * __uint_as_float(v[j + 2]), p.alpha * __uint_as_float(v[j + 3]));
                    } else {
#pragma unroll
                        for (int j = 0; j < 32; ++j) {
                            if (nb + j < p.N) {
                                float o = p.alpha * __uint_as_float(v[j]);
                                if (p.beta != 0.f) o += p.beta * d[j];
                                d[j] = o;
                            }
                        }
                    }
                }
            }
            };  // drain one 128-row half
            for (int hh = 0; hh < p.mt; ++hh) drain(hh);
            // release this accumulator to the MMA warp
            tc_fence_before();
            __syncwarp();
            if (lane == 0) mbar_arrive(smem_u32(&tempty[acc]));
            if (++acc == p.nacc) { acc = 0; aph ^= 1u; }
        }
    }
    if constexpr (SPLITK) {
        if (p.cl) {
            // Deterministic split-K reduction: every CTA of the
            // cluster holds one split's alpha-scaled partial tile in shared memory; CTA
            // rank rho sums rows [rho*rows_per, ...) of all cl partials over DSMEM in rank
            // order and writes them to dw (split group 0 applies beta; later groups add
            // in group order behind a turn counter per (tile, slab)).
            asm volatile("barrier.cluster.arrive.release;\n\tbarrier.cluster.wait.acquire;" ::: "memory");
            {
                // all 288 threads of the CTA share its slab (the mainloop is over)
                const int ep = threadIdx.x;
                const int rho = blockIdx.x % p.cl, c = blockIdx.x / p.cl;
                const int nbatch = p.zsplit ? p.num_z / p.zsplit : 1;
                const int nu = per_z * nbatch;
                const int g = g_ticket >= 0 ? g_ticket : c / nu, u = c % nu;
                const int batch = u / per_z, rem = u - batch * per_z;
                const int ntile = rem / mt;
                const int m0 = (rem - ntile * mt) * BMt, n0 = ntile * p.BN;
                const int rows_per = (BMt + p.cl - 1) / p.cl;
                const int r0 = rho * rows_per, r1 = min(BMt, r0 + rows_per);
                const int nq = p.BN / 4;
                const int pitch = p.BN + 4;
                const float bsplit = g == 0 ? p.beta : 1.f;
                // NEXT-3: the last split group writes the final dw: it also adds the
                // cross-rank sum through the multicast address
                const bool final_mc = p.red.n != 0 && g == p.red_group;
                unsigned long long* turn =
                    p.turns ? p.turns + ((size_t)(batch * per_z + rem) * p.cl + rho) : nullptr;
                const uint32_t stg = smem_u32(smem);
                float* outF = (float*)p.out + (p.zsplit ? (size_t)batch * p.batch_stride : 0);
                // thread -> (column quad c4, row phase rsub): one division per thread
                const int tpr = (int)blockDim.x / nq;  // rows in flight per pass
                const bool active = ep < tpr * nq;
                const int c4 = ep % nq, rsub = ep / nq;
                const int col0 = n0 + 4 * c4;
                uint32_t part[16];  // this slab position in every partner's shared memory
#pragma unroll
                for (int k = 0; k < 16; ++k) {
                    part[k] = 0;
                    if (k < p.cl) asm("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(part[k]) : "r"(stg), "r"(k));
                }
                constexpr int U = 8;  // rows per thread per batch (loads in flight)
                // this split group's turn: groups add into dw in order
                if (turn && g > 0) {
                    if (ep == 0) turn_wait(turn, turn_tag(p.epoch, g - 1));
                    __syncthreads();
                }
                for (int rb = r0 + rsub; rb < r1; rb += U * tpr) {
                    // 1. the cluster's partials of these rows, summed in rank order (a fixed
                    //    order: deterministic)
                    float4 sum[U];
#pragma unroll
                    for (int uu = 0; uu < U; ++uu) sum[uu] = make_float4(0.f, 0.f, 0.f, 0.f);
                    for (int k = 0; k < p.cl; ++k) {
#pragma unroll
                        for (int uu = 0; uu < U; ++uu) {
                            const int rr = rb + uu * tpr;
                            if (!active || rr >= r1) continue;
                            float q0, q1, q2, q3;
                            asm volatile("ld.shared::cluster.v4.f32 {%0, %1, %2, %3}, [%4];"
                                         : "=f"(q0), "=f"(q1), "=f"(q2), "=f"(q3)
                                         : "r"(part[k] + (uint32_t)((rr * pitch + 4 * c4) * 4)));
                            sum[uu].x += q0; sum[uu].y += q1; sum[uu].z += q2; sum[uu].w += q3;
                        }
                    }
                    // 2. dw = sum + bsplit * dw: all loads of the batch, then the stores
                    if (active) {
                        if constexpr (EPI == EPI_WGRAD_CHAIN) {
                            const bool vec = col0 + 3 < p.N && (p.ldc & 3) == 0 && ((((uintptr_t)outF) & 15) == 0);
                            float4 old[U];
#pragma unroll
                            for (int uu = 0; uu < U; ++uu) {
                                const int rr = rb + uu * tpr;
                                old[uu] = make_float4(0.f, 0.f, 0.f, 0.f);
                                if (rr >= r1 || m0 + rr >= p.M || bsplit == 0.f) continue;
                                const float* d = outF + (size_t)(m0 + rr) * p.ldc + col0;
                                if (vec) {
                                    old[uu] = __ldcg(reinterpret_cast<const float4*>(d));
                                } else {
                                    old[uu].x = col0 < p.N ? __ldcg(d) : 0.f;
                                    old[uu].y = col0 + 1 < p.N ? __ldcg(d + 1) : 0.f;
                                    old[uu].z = col0 + 2 < p.N ? __ldcg(d + 2) : 0.f;
                                    old[uu].w = col0 + 3 < p.N ? __ldcg(d + 3) : 0.f;
                                }
                            }
#pragma unroll
                            for (int uu = 0; uu < U; ++uu) {
                                const int rr = rb + uu * tpr;
                                if (rr >= r1 || m0 + rr >= p.M) continue;
                                float* d = outF + (size_t)(m0 + rr) * p.ldc + col0;
                                const float4 o = make_float4(sum[uu].x + bsplit * old[uu].x, sum[uu].y + bsplit * old[uu].y,
                                                             sum[uu].z + bsplit * old[uu].z, sum[uu].w + bsplit * old[uu].w);
                                const long long ro = (long long)(d - (const float*)p.out);
                                if (vec) {
                                    *reinterpret_cast<float4*>(d) = o;
                                    if (final_mc) red_add4(p.red, ro, o);
                                } else {
                                    if (col0 < p.N) d[0] = o.x;
                                    if (col0 + 1 < p.N) d[1] = o.y;
                                    if (col0 + 2 < p.N) d[2] = o.z;
                                    if (col0 + 3 < p.N) d[3] = o.w;
                                    if (final_mc) {
                                        if (col0 < p.N) red_add(p.red, ro, o.x);
                                        if (col0 + 1 < p.N) red_add(p.red, ro + 1, o.y);
                                        if (col0 + 2 < p.N) red_add(p.red, ro + 2, o.z);
                                        if (col0 + 3 < p.N) red_add(p.red, ro + 3, o.w);
                                    }
                                }
                            }
                        } else {
                            // scattered layouts (small-C, space-to-depth, window): per element
#pragma unroll
                            for (int uu = 0; uu < U; ++uu) {
                                const int rr = rb + uu * tpr;
                                if (rr >= r1 || m0 + rr >= p.M) continue;
                                const float sv[4] = {sum[uu].x, sum[uu].y, sum[uu].z, sum[uu].w};
                                long long o[4];
                                float ov[4];
#pragma unroll
                                for (int j = 0; j < 4; ++j) {
                                    o[j] = col0 + j < p.N ? wgrad_dst<EPI, ELT>(p, m0 + rr, col0 + j) : -1;
                                    ov[j] = (bsplit != 0.f && o[j] >= 0) ? __ldcg(outF + o[j]) : 0.f;
                                }
#pragma unroll
                                for (int j = 0; j < 4; ++j)
                                    if (o[j] >= 0) {
                                        const float fv = sv[j] + bsplit * ov[j];
                                        outF[o[j]] = fv;
                                        if (final_mc) red_add(p.red, (long long)(outF + o[j] - (const float*)p.out), fv);
                                    }
                            }
                        }
                    }
                }
                if (turn) {
                    __syncthreads();
                    if (ep == 0) turn_post(turn, turn_tag(p.epoch, g));
                }
            }
            // partners may still be reading this CTA's staging
            asm volatile("barrier.cluster.arrive.release;\n\tbarrier.cluster.wait.acquire;" ::: "memory");
        }
    }
    tc_fence_before();
    __syncthreads();
    if (warp == 4) {
        tc_fence_after();
        asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(p.tmem_cols));
    }
}
