/*
 * mucudnn.h -- C ABI of the B200-native micro-batched convolution library
 * (the hot path of mu-cuDNN: Oyama, Ben-Nun, Hoefler, Matsuoka, IEEE CLUSTER
 * 2018; text in /root/reference/PAPER.md, cited as P:Lnn = line nn).
 *
 * What the library does (north_star of BASELINE.json):
 *   A convolution layer's mini-batch of N samples is split into micro-batches
 *   (Sec. II/III, Fig. 3).  Each micro-batch is executed with
 *   one of three equivalent sm_100a convolution algorithms that trade
 *   workspace for speed: implicit GEMM (zero workspace), explicit
 *   im2col + GEMM, Winograd F(2x2,3x3).  A benchmark pass times every
 *   (algorithm, micro-batch size) pair (WR step 1); a dynamic program
 *   picks the partition of N and per-part algorithm minimising the total time
 *   within a per-layer workspace limit (WR policy, Sec. III-B); a
 *   set-valued DP + Pareto pruning + exact multiple-choice-knapsack solve the
 *   whole-network shared-workspace problem (WD policy, Sec. III-C,
 *   ILP Eq. (1)-(4)).  Plans are executed on the caller's CUDA stream and
 *   workspace.
 *
 * Conventions (all functions):
 *   - Every function returns mucu_status_t; none throws, aborts or prints.
 *     On error, mucu_last_error(handle) returns a thread-local detail string.
 *   - Tensors: activations NHWC (x: [N,H,W,C], y/dy: [N,P,Q,K], dx: [N,H,W,C]),
 *     filters KRSC (w: [K,R,S,C]), all densely packed.  Element type by math
 *     mode: MUCU_MATH_F32 / MUCU_MATH_TF32 -> float32; MUCU_MATH_BF16 ->
 *     bfloat16.  The filter gradient dw is ALWAYS float32 [K,R,S,C].
 *     P = (H + 2 pad - R)/stride + 1, Q likewise (reading G1/G3).
 *   - Device memory (tensors, workspace, benchmark scratch) is owned by the
 *     caller (PyTorch allocator); the library never calls cudaMalloc.  Host
 *     objects (handle, network) are created and destroyed by the library.
 *     BackwardFilter's split-K ordering counters live in a static device array
 *     of the library module (2 MiB, no allocation call).
 *   - GPU work is asynchronous on the caller's `cuda_stream` (a cudaStream_t
 *     passed as void*; NULL = legacy default stream), except
 *     mucu_benchmark / mucu_plan_layer / mucu_network_plan which synchronise
 *     that stream before returning.
 *   - Pure host functions (marked "host") never touch the GPU and are
 *     reentrant.  A handle is not thread-safe; use one per host thread.
 */
#ifndef MUCUDNN_H_
#define MUCUDNN_H_

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define MUCU_VERSION 100 /* 1.0.0 */

typedef enum {
    MUCU_OK = 0,
    MUCU_ERR_INVALID_VALUE = 1,          /* bad dims, null pointer, plan parts not summing to N */
    MUCU_ERR_UNSUPPORTED = 2,            /* algorithm ineligible for this layer/type (e.g. WG on 5x5) */
    MUCU_ERR_INSUFFICIENT_WORKSPACE = 3, /* ws_bytes below what the plan needs / nothing fits the limit */
    MUCU_ERR_INFEASIBLE = 4,             /* WD budget below the sum of minimal workspaces */
    MUCU_ERR_CAPACITY = 5,               /* caller array too small; *count holds the needed size */
    MUCU_ERR_MISALIGNED = 6,             /* device pointer not 16-byte aligned */
    MUCU_ERR_CUDA = 7,                   /* CUDA runtime/driver error (message in mucu_last_error) */
    MUCU_ERR_INTERNAL = 8
} mucu_status_t;

/* The three convolution operations of cuDNN. */
typedef enum { MUCU_FWD = 0, MUCU_BWD_DATA = 1, MUCU_BWD_FILTER = 2 } mucu_conv_type_t;

/* Algorithms; the enum order is the tie-break order (reading G11). */
typedef enum {
    MUCU_ALGO_IMPLICIT_GEMM = 0,     /* (a) zero workspace                                   */
    MUCU_ALGO_IM2COL_GEMM = 1,       /* (b) explicit im2col (+col2im for DGRAD) + GEMM        */
    MUCU_ALGO_WINOGRAD_2X2_3X3 = 2,  /* (c) Winograd F(2x2,3x3), Lavin & Gray (ref [23])      */
    MUCU_ALGO_FFT = 3,               /* (d) frequency domain, one F x F tile per image         */
    MUCU_ALGO_FFT_TILING = 4,        /* (e) frequency domain on 32 x 32 tiles   */
    MUCU_NUM_ALGOS = 5
} mucu_algo_t;

/* Arithmetic: F32 = fp32 SIMT FFMA; TF32 = fp32 storage, tcgen05 kind::tf32;
 * BF16 = bf16 storage, tcgen05 kind::f16 (bf16 x bf16 -> fp32 in TMEM). */
typedef enum { MUCU_MATH_F32 = 0, MUCU_MATH_TF32 = 1, MUCU_MATH_BF16 = 2 } mucu_math_t;

/* Batch-size policies of P:L149-155: which micro-batch sizes b are benchmarked.
 * ALL: b = 1..N.  POW2: {2^k <= N} U {N} (reading G20).  UNDIVIDED: {N}. */
typedef enum { MUCU_POLICY_ALL = 0, MUCU_POLICY_POW2 = 1, MUCU_POLICY_UNDIVIDED = 2 } mucu_policy_t;

/* Layer descriptor (north_star: N,C,H,W,K,R,S,pad,stride; dilation 1, groups 1). */
typedef struct {
    int32_t n, c, h, w, k, r, s, pad, stride;
    int32_t math; /* mucu_math_t */
} mucu_conv_desc_t;

/* Micro-configuration: an (algorithm, micro-batch size) pair.  A
 * configuration / plan is an array of these; its micro_n sum to desc.n and it
 * is executed in array order (reading G8: non-increasing micro_n). */
typedef struct {
    int32_t algo;
    int32_t micro_n;
} mucu_micro_config_t;

typedef struct mucu_handle* mucu_handle_t;   /* library-owned, one per device */
typedef struct mucu_network* mucu_network_t; /* library-owned WD kernel list */

/* ---------------------------------------------------------------- misc ---- */
const char* mucu_status_string(mucu_status_t status);   /* host; static string */
/* host; detail of the calling thread's last error (thread-local; `handle` may
 * be NULL, e.g. after a failed pure host function or mucu_create). */
const char* mucu_last_error(mucu_handle_t handle);
int32_t mucu_version(void);                             /* host */
/* Process-wide number of CUDA kernels the library has launched so far (host;
 * monotone, for launch accounting in benchmarks). */
uint64_t mucu_launch_count(void);

/* Create a handle bound to CUDA device `device` (makes it current on the
 * calling thread).  Reads env MUCU_BATCH_POLICY={all,pow2,undivided} (default
 * pow2), MUCU_BENCH_WARMUP (default 2), MUCU_BENCH_REPS (default 5). */
mucu_status_t mucu_create(mucu_handle_t* handle, int device);
mucu_status_t mucu_destroy(mucu_handle_t handle);
/* the batch-size policy "can be specified via an environment variable
 * or through a special library function" -- this is the function. */
mucu_status_t mucu_set_policy(mucu_handle_t handle, mucu_policy_t policy);
mucu_status_t mucu_set_bench_params(mucu_handle_t handle, int32_t warmup, int32_t reps);
/* BackwardFilter reduction order (dW is a plain sum over samples).
 * deterministic = 1 (default; env MUCU_DETERMINISTIC): when a kernel splits the
 * pixel reduction of a dw tile over several CTAs, the partials are combined in a
 * fixed order (a thread-block cluster sums its CTAs' partials over distributed
 * shared memory in rank order; split groups add into dw in group order behind a
 * turn counter), so dw is bitwise reproducible run to run.  deterministic = 0:
 * every split adds its partial with fp32 L2 reductions (faster on layers with
 * few dw tiles and long reductions; run-to-run rounding differences).  FWD and
 * BackwardData are deterministic in both modes.  Results of either mode equal
 * the exact sum within fp32 rounding; integer-valued data are exact. */
mucu_status_t mucu_set_deterministic(mucu_handle_t handle, int32_t deterministic);

/* ------------------------------------------------------ host: geometry ---- */
/* P and Q of the output (host).  INVALID_VALUE if any dim <= 0 or P,Q <= 0. */
mucu_status_t mucu_output_dims(const mucu_conv_desc_t* desc, int32_t* p, int32_t* q);

/* Exact workspace bytes of one micro-configuration (host; "within the
 * workspace constraint").  Closed forms (elt = 4 for F32/TF32, 2 for BF16,
 * every segment rounded up to 256 B):
 *   IG  (all types):  0
 *   I2C FWD/WGRAD:    b*P*Q*ceil_e(R*S*C)*elt  (+ K*ceil_e(R*S*C)*elt when R*S*C*elt % 16 != 0)
 *                     0 for 1x1, stride 1, pad 0 (the im2col matrix is x itself)
 *                     b*H*W*16 for TF32/BF16 with C*elt < 16 (RGB input layer): x with
 *                     channels zero-padded to 16 B, gathered tap by tap on chip
 *                     TF32/BF16 WGRAD adds Ps partial dW slots of K*R*S*C*4 bytes (deterministic
 *                     split-K summed in split order; 0 when Ps = 1):
 *                       Ps = min(148, ceil(148 / (ceil(K/128) * ceil(R*S*C/128))));
 *                     and when C is a multiple of 128/elt (not 1x1) the im2col is done by TMA
 *                     into shared memory: only the slots, with
 *                       Ps = min(148, ceil(148 / (ceil(K/256) * ceil(R*S*C/256))))
 *   I2C DGRAD:        b*P*Q*ceil_4(R*S*C)*4 (fp32 dcol)  (+ filter copy as above, or with rows of
 *                     128 B when R*S*C < 128/elt on tensor cores); 0 for 1x1/s1/p0
 *   I2C, TF32/BF16, stride st > 1 and C*elt < 16 ("space-to-depth"):
 *                     FWD: u = 2, f = st*u, Dr = (st*(u-1) + R - 1)/f + 1, Ds likewise,
 *                          Cs = f*f*C rounded up to 128/elt, Pu = ceil(P/u), Qu = ceil(Q/u):
 *                          u*u*K*Dr*Ds*Cs*elt + b*(Pu+Dr-1)*(Qu+Ds-1)*Cs*elt
 *                     WGRAD when the staged-row kernel applies (C*elt < 16, R*S*C <= 512,
 *                          K <= 256 and a multiple of 128/elt, the x row W*C*elt splits into 16-B-multiple
 *                          chunks, TR - R*S*C <= R*S*C/4): 148 partial dW tiles, TR = R*S*C rounded up to 128:
 *                          148 * TR * K * 4  (b-independent; split order fixed: deterministic)
 *                     else WGRAD with C <= 4 and st*16 % 16 == 0 (BF16: st even) ("window"):
 *                          b*H*Wp*4*elt; atoms of aw bytes (TF32: 128; BF16: the aw in {128, 64, 32}
 *                          minimising align256(R*na*aw/elt), larger aw on ties), tpa = aw/(4*elt)
 *                          taps per atom, na = ceil(S/tpa), Wp = max(st*(Q-1) + na*tpa, W + pad)
 *                          rounded up to 4; + 148 partial dW tiles of M = R*na*aw/elt window rows:
 *                          align256(148 * M * K * 4) (deterministic split-K in split order)
 *                     WGRAD otherwise (u = 1, f = st): b*(P+Dr-1)*(Q+Ds-1)*Cs*elt
 *                     DGRAD (when K % (128/elt) == 0, st*st*C <= 256): u = 2 if (2*st)^2*C <= 256
 *                          else 1, f = st*u, Dr = ceil(R/st) - 1 + u, Ds likewise: f*f*C*Dr*Ds*K*elt
 *   WG  FWD:          16*K*C*elt + 16*b*T*C*elt + 16*b*T*K*4,   T = ceil(P/2)*ceil(Q/2)
 *   WG  DGRAD:        16*C*K*elt + 16*b*T'*K*elt + 16*b*T'*C*4, T' = ceil(H/2)*ceil(W/2)
 *   WG  WGRAD:        F(3x3,2x2), Tp = b*T rounded up to 256, Cp / Kp = C / K
 *                     rounded up to 128/elt:  16*Tp*Cp*elt + 16*Tp*Kp*elt + 16*Kp*Cp*4
 *   FFT / FFT_TILING (F32 only, stride 1): complex spectra of B = F*(F/2+1)
 *                     bins, 8 bytes per value, planes Pl = b*ty*tx tiles.  Output grid E = P x Q
 *                     (FWD, WGRAD) or H x W (DGRAD); FFT: one tile per image, F = the smallest
 *                     power of two >= max(Eh + R - 1, Ew + S - 1), 8 <= F <= 32; FFT_TILING:
 *                     F = 32, tiles of min(Eh, 33-R) x min(Ew, 33-S) outputs (R, S <= 16),
 *                     ty x tx = ceil(Eh/Th) x ceil(Ew/Tw):
 *                     FWD:   8*B*K*C + 8*B*Pl*C + 8*B*Pl*K
 *                     DGRAD: 8*B*K*C + 8*B*Pl*K + 8*B*Pl*C
 *                     WGRAD: 8*B*K*C (the dW spectrum, first) + 8*B*Pl*C + 8*B*Pl*K
 * ceil_e rounds up to a multiple of 16/elt elements.  UNSUPPORTED if the
 * algorithm is ineligible (WG needs R=S=3, stride 1, pad <= 2; FFT / FFT_TILING
 * need MUCU_MATH_F32 and stride 1). */
mucu_status_t mucu_workspace_size(const mucu_conv_desc_t* desc, mucu_conv_type_t type,
                                  mucu_algo_t algo, int32_t micro_n, uint64_t* bytes);

/* ---------------------------------------------------- host: optimisers ---- */
/* Timing tables (P:L88 step 1): time_ns and ws are row-major
 * [MUCU_NUM_ALGOS][n+1]; entry [a][b] is the time (ns, int64) and workspace
 * (bytes) of algorithm a at micro-batch b; time < 0 = not benchmarked /
 * ineligible; column b = 0 is ignored. */

/* WR dynamic program (Sec. III-B):
 *   T(b) = min( T_mu(b), min_{1<=b'<b} T_mu(b') + T(b-b') ),  T(0) = 0,
 * T_mu(b) = fastest present entry with ws <= ws_limit (ties: smaller ws, then
 * smaller algo id; reading G11).  Canonical tie-break among optimal plans
 * (reading G8): fewer micro-batches, then parts sorted non-increasing and
 * compared lexicographically larger-first.  Output: *count micro-configs in
 * out[0..cap) in non-increasing micro_n, *total_ns = T(n).
 * Errors: INSUFFICIENT_WORKSPACE if no plan fits; CAPACITY if cap < count. */
mucu_status_t mucu_plan_wr(int32_t n, const int64_t* time_ns, const uint64_t* ws, uint64_t ws_limit,
                           mucu_micro_config_t* out, int32_t cap, int32_t* count, int64_t* total_ns);

/* WD desirable set of one kernel (Sec. III-C1): the set-valued DP
 *   C(b) = D( U_{1<=b'<=b} { [c] (+) C' : c in C_mu(b'), C' in C(b-b') } ),  C(0) = {[]}
 * with T = sum of times, M = max of workspaces (reading G13) and D the Pareto
 * filter "keep C iff no other configuration is at least as fast with no more
 * workspace" (reading G15).  Only micro-configs with ws <= ws_cap take part.
 * Output sorted by M ascending (T strictly decreasing): front_t[i], front_m[i],
 * and one plan per point in plans[i*n .. i*n + plan_len[i]) (valid, not
 * necessarily unique among equal-cost plans).  CAPACITY if cap < *front_len. */
mucu_status_t mucu_pareto_front(int32_t n, const int64_t* time_ns, const uint64_t* ws, uint64_t ws_cap,
                                int64_t* front_t, uint64_t* front_m, int32_t cap, int32_t* front_len,
                                mucu_micro_config_t* plans, int32_t* plan_len);

/* WD 0-1 ILP (Eq. (1)-(4)) as an exact multiple-choice knapsack:
 *   min sum_k t_k(c_k)  s.t.  sum_k align256(m_k(c_k)) <= total_limit, one c per kernel.
 * Options of kernel k are t[off_k .. off_k+front_len[k]), m[...] with off_k the
 * prefix sum of front_len.  Ties: smaller sum of aligned m, then the
 * lexicographically smallest choice vector (reading G17).  Output choice[k],
 * offset[k] (byte offset of kernel k's segment = running sum of aligned m in
 * kernel order, reading G18), *total_ns.  INFEASIBLE if even the smallest
 * options exceed total_limit. */
mucu_status_t mucu_solve_wd(int32_t num_kernels, const int32_t* front_len, const int64_t* t,
                            const uint64_t* m, uint64_t total_limit, int32_t* choice,
                            uint64_t* offset, int64_t* total_ns);

/* ------------------------------------------------------------- GPU ---- */
/* Benchmark pass (P:L88 WR step 1): for every b in the handle's policy set and
 * every eligible algorithm whose workspace fits ws_limit, run the micro-config
 * on scratch tensors: `warmup` launches (the last one timed), then three
 * CUDA-event samples, each the mean of up to `reps` back-to-back launches (the
 * way a plan's micro-batches run; a sample stops at ~1 ms of work, so a long
 * micro-config takes one launch per sample), median of the three, quantised to
 * ns (reading G21).  Steady state: the
 * b-independent workspace prefix (filter transforms) is computed by the warm-up
 * and reused, as the executor computes it once per call.  Fills time_ns / ws
 * ([MUCU_NUM_ALGOS][desc->n + 1], -1 / 0 where not measured).  Identical
 * requests are served from the handle's in-memory cache.
 * scratch: device buffer of >= mucu_benchmark_scratch_size() bytes (contents
 * overwritten; the caller may pre-fill it with data of its choice).
 * Synchronises cuda_stream. */
mucu_status_t mucu_benchmark_scratch_size(const mucu_conv_desc_t* desc, mucu_conv_type_t type,
                                          uint64_t ws_limit, uint64_t* bytes);
mucu_status_t mucu_benchmark(mucu_handle_t handle, const mucu_conv_desc_t* desc, mucu_conv_type_t type,
                             uint64_t ws_limit, void* scratch, uint64_t scratch_bytes, void* cuda_stream,
                             int64_t* time_ns, uint64_t* ws);

/* WR convenience: mucu_benchmark + mucu_plan_wr (P:L86-92 steps 1-3). */
mucu_status_t mucu_plan_layer(mucu_handle_t handle, const mucu_conv_desc_t* desc, mucu_conv_type_t type,
                              uint64_t ws_limit, void* scratch, uint64_t scratch_bytes, void* cuda_stream,
                              mucu_micro_config_t* out, int32_t cap, int32_t* count, int64_t* total_ns);

/* Execute a plan (Fig. 3): for each micro-config in order, offset
 * the activation pointers by the samples already done and run the algorithm on
 * micro_n samples.  out = alpha * op + beta * out (reading G5).
 *   forward:          (x, w) -> y
 *   backward_data:    (dy, w) -> dx
 *   backward_filter:  (x, dy) -> dw (fp32); the user's beta applies to the
 *                     first micro-batch, later ones accumulate with beta = 1
 *                     ("output scale", reading G5).
 * workspace: device buffer of ws_bytes >= max over the plan of
 * mucu_workspace_size (INSUFFICIENT_WORKSPACE otherwise; NULL allowed when 0).
 * Asynchronous on cuda_stream.  All device pointers must be 16-byte aligned. */
mucu_status_t mucu_conv_forward(mucu_handle_t handle, const mucu_conv_desc_t* desc,
                                const mucu_micro_config_t* plan, int32_t count, float alpha,
                                const void* x, const void* w, float beta, void* y,
                                void* workspace, uint64_t ws_bytes, void* cuda_stream);
mucu_status_t mucu_conv_backward_data(mucu_handle_t handle, const mucu_conv_desc_t* desc,
                                      const mucu_micro_config_t* plan, int32_t count, float alpha,
                                      const void* dy, const void* w, float beta, void* dx,
                                      void* workspace, uint64_t ws_bytes, void* cuda_stream);
mucu_status_t mucu_conv_backward_filter(mucu_handle_t handle, const mucu_conv_desc_t* desc,
                                        const mucu_micro_config_t* plan, int32_t count, float alpha,
                                        const void* x, const void* dy, float beta, float* dw,
                                        void* workspace, uint64_t ws_bytes, void* cuda_stream);

/* ------------------------------------------- NEXT-3: fused dW reduction ---- */
/* Data-parallel training sums every layer's dW over the ranks (micro-
 * batching lets "the communication of parameter gradients" be hidden; SURVEY
 * 8(f) NEXT-3).  Here the sum is fused into BackwardFilter: the kernel that
 * writes a dw element's final value (the last micro-batch's epilogue, its last
 * ordered split group, or the partial-slot reduction; one push kernel after the
 * F32 SIMT / Winograd / FFT / atomic split-K writers) also adds it to a
 * reduction target, element-aligned with dw:
 *   multicast = 1, count = 1: dst[0] is the NVLink multicast address of a
 *     symmetric fp32 buffer (mucu_nvls_*): one multimem.red.add.f32 per value,
 *     NVSwitch adds it into every rank's copy;
 *   multicast = 0, count = ranks: dst[r] is rank r's buffer (a peer pointer over
 *     NVLink P2P, or this rank's own): one red.global.add.f32 per rank.
 * Protocol per iteration: zero this rank's buffer, barrier, every rank's
 * backward_filter_reduce calls, barrier; then every rank's buffer holds the sum
 * over ranks of dw.  Additions arrive in any order (exact for 2 ranks, since
 * 0 + a + b = 0 + b + a; flush-to-zero like every fp32 reduction).
 * Errors: INVALID_VALUE (count outside 1..MUCU_MAX_REDUCE_RANKS, multicast with
 * count != 1), MISALIGNED (a dst NULL or not 16-byte aligned), else as
 * mucu_conv_backward_filter. */
#define MUCU_MAX_REDUCE_RANKS 8
typedef struct {
    int32_t multicast;
    int32_t count;
    float* dst[MUCU_MAX_REDUCE_RANKS];
} mucu_reduce_target_t;
/* dw (device, this rank's) receives exactly what mucu_conv_backward_filter
 * computes; the target receives += the same final values. */
mucu_status_t mucu_conv_backward_filter_reduce(mucu_handle_t handle, const mucu_conv_desc_t* desc,
                                               const mucu_micro_config_t* plan, int32_t count, float alpha,
                                               const void* x, const void* dy, float beta, float* dw,
                                               const mucu_reduce_target_t* target, void* workspace,
                                               uint64_t ws_bytes, void* cuda_stream);
/* Device-side barrier over the ranks, enqueued on cuda_stream: a system-scope
 * release of this rank's earlier reductions, +1 on every flag word of `flags`
 * (uint32 words cast to float*: one multicast address, or every rank's flag),
 * then a wait until *own (this rank's flag, device) >= target (= ranks x
 * barriers so far; every rank calls it equally often).  A wait longer than 10 s
 * traps (the stream reports a CUDA error) instead of hanging. */
mucu_status_t mucu_peer_barrier(const mucu_reduce_target_t* flags, const uint32_t* own, uint32_t target,
                                void* cuda_stream);

/* NVLink multicast object, one per rank (device = this rank's CUDA device,
 * ranks = world size, bytes = user bytes; all ranks pass the same values):
 *   rank 0: mucu_nvls_create, mucu_nvls_export -> a POSIX fd owned by the
 *           caller, passed to the peers (pidfd_getfd);
 *   others: mucu_nvls_import(fd);
 *   all:    mucu_nvls_bind -> local (this rank's copy, unicast) and multicast
 *           addresses of the user bytes; blocks until every rank has created or
 *           imported; the buffer starts zeroed.
 * mucu_nvls_barrier(stream): mucu_peer_barrier on the object's own flag word.
 * Errors: UNSUPPORTED (no multicast on the device), CUDA (driver call failed,
 *   e.g. no NVSwitch fabric; detail in mucu_last_error), INVALID_VALUE. */
typedef struct mucu_nvls* mucu_nvls_t;
mucu_status_t mucu_nvls_supported(int device, int32_t* supported);     /* host */
mucu_status_t mucu_nvls_create(int device, int32_t ranks, uint64_t bytes, mucu_nvls_t* out);
mucu_status_t mucu_nvls_export(mucu_nvls_t nv, int32_t* fd);
mucu_status_t mucu_nvls_import(int device, int32_t ranks, uint64_t bytes, int32_t fd, mucu_nvls_t* out);
mucu_status_t mucu_nvls_bind(mucu_nvls_t nv, void** local, void** multicast);
mucu_status_t mucu_nvls_barrier(mucu_nvls_t nv, void* cuda_stream);
mucu_status_t mucu_nvls_destroy(mucu_nvls_t nv);

/* ------------------------------------------------------------ WD ---- */
/* WD needs every kernel before optimising: register the kernels,
 * then plan once.  mucu_network_plan benchmarks each unique (desc, type)
 * (deduplicated), builds each kernel's desirable set with the
 * set-valued DP (ws_cap = total_limit) and solves the MCKP.  Then
 * mucu_network_get returns kernel `kernel_id`'s plan, its segment offset into
 * the caller's single network workspace and the segment size. */
mucu_status_t mucu_network_create(mucu_network_t* net);
mucu_status_t mucu_network_destroy(mucu_network_t net);
mucu_status_t mucu_network_add(mucu_network_t net, const mucu_conv_desc_t* desc, mucu_conv_type_t type,
                               int32_t* kernel_id);
mucu_status_t mucu_network_plan(mucu_network_t net, mucu_handle_t handle, uint64_t total_limit,
                                void* scratch, uint64_t scratch_bytes, void* cuda_stream);
/* Same as mucu_network_plan but from caller-supplied timing tables (one
 * [MUCU_NUM_ALGOS][n_k+1] pair per kernel, concatenated in kernel order);
 * host-only, for offline planning from a stored benchmark table. */
mucu_status_t mucu_network_plan_from_tables(mucu_network_t net, uint64_t total_limit,
                                            const int64_t* time_ns, const uint64_t* ws);
mucu_status_t mucu_network_get(mucu_network_t net, int32_t kernel_id, mucu_micro_config_t* out,
                               int32_t cap, int32_t* count, uint64_t* ws_offset, uint64_t* ws_bytes,
                               int64_t* time_ns);

#ifdef __cplusplus
}
#endif
#endif /* MUCUDNN_H_ */
