// api.cu -- C ABI (include/bzk.h), batch scheduler (waves, ping-pong scratch, tail cut-off) and
// stream loader (host -> device waves on a side stream, "dynamic loading").
//
// a1 input residency/loading, a8 batch scheduler; the kernels for rows
// a2-a7 live in sumcheck.cuh.
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#include <algorithm>
#include <string>
#include <vector>

#include <cudaTypedefs.h>
#include <nvtx3/nvToolsExt.h>

#include "bzk.h"
#include "field.cuh"
#include "field_f64.cuh"
#include "gl.cuh"
#include "gen.cuh"
#include "merkle.cuh"
#include "multiround.cuh"
#include "small.cuh"
#include "encoder.cuh"
#include "sha256.cuh"
#include "sumcheck.cuh"

using namespace bzk;

namespace {

constexpr uint32_t kThreads = 256;
constexpr uint32_t kRoundThreads = BZK_RT;   // k_round CTA size (sumcheck.cuh)
constexpr uint32_t kTailLog = 8;          // rounds with h <= 2^kTailLog pairs run in k_tail
constexpr uint32_t kSMs = 148;

struct ProfRec { int kind; cudaEvent_t a, b; };

// NVTX ranges (host timeline for nsys: calls, jobs, waves, stage chains), on when BZK_NVTX=1.
// nvtx3 is header-only: without a profiler attached the calls are no-ops.
bool nvtx_on() {
    static const bool on = [] { const char *e = getenv("BZK_NVTX"); return e && atoi(e) != 0; }();
    return on;
}
struct NvtxRange {
    bool active;
    explicit NvtxRange(const char *name) : active(nvtx_on()) { if (active) nvtxRangePushA(name); }
    ~NvtxRange() { if (active) nvtxRangePop(); }
};

}  // namespace

struct bzk_ctx {
    int device = 0;
    size_t workspace_limit = 0;
    void *ws = nullptr;
    size_t ws_size = 0;
    cudaStream_t copy_stream = nullptr;
    cudaEvent_t ev_copied[2] = {nullptr, nullptr};
    cudaEvent_t ev_consumed[2] = {nullptr, nullptr};
    // Merkle loader (NEXT-3): device->host stream for node levels, per-slot events
    cudaStream_t d2h_stream = nullptr;
    cudaEvent_t ev_nodes_ready[2] = {nullptr, nullptr};
    cudaEvent_t ev_nodes_copied[2] = {nullptr, nullptr};
    // loader ring: two device staging slots for host tables, reused across waves, jobs and calls
    void *stage[2] = {nullptr, nullptr};
    size_t stage_size = 0;
    int next_slot = 0;
    bool slot_used[2] = {false, false};
    uint32_t *d_flag = nullptr;
    fe *consts = nullptr;            // Lagrange / node constants (k_init_consts)
    std::string last_error;
    bool prof = false;
    std::vector<ProfRec> recs;
    std::vector<cudaEvent_t> ev_pool;
    uint64_t launches = 0;
    int num_sms = kSMs;
    size_t auto_limit = 0;           // cached default workspace limit (0 = recompute)
    // CUDA graph of the last BZK_F_GRAPH call, replayed while the submitted jobs are identical
    cudaGraphExec_t graph_exec = nullptr;
    std::vector<unsigned char> graph_key;
    uint64_t graph_launches = 0;      // kernel launches inside the cached graph
    // end of the context's last call: every call first waits on it, so calls issued on different
    // streams never overlap on the shared workspace (ps, tickets, partials, ping-pong buffers)
    cudaEvent_t ev_done = nullptr;
    bool ev_done_recorded = false;
    // bzk_commit_prove's module pipeline: Merkle and sum-check side streams, Merkle stage scratch
    cudaStream_t chain_mk = nullptr, chain_sc = nullptr;
    cudaStream_t dual_stream = nullptr;
    void *chain_ws = nullptr;
    size_t chain_ws_size = 0;
};

namespace {

bzk_status fail(bzk_ctx *c, bzk_status s, const std::string &msg) {
    if (c) c->last_error = msg;
    return s;
}

bzk_status cuda_fail(bzk_ctx *c, cudaError_t e, const char *where) {
    return fail(c, BZK_ECUDA, std::string(where) + ": " + cudaGetErrorString(e));
}

#define CK(call)                                                   \
    do {                                                           \
        cudaError_t _e = (call);                                   \
        if (_e != cudaSuccess) return cuda_fail(ctx, _e, #call);   \
    } while (0)

cudaEvent_t pool_event(bzk_ctx *ctx) {
    if (!ctx->ev_pool.empty()) {
        cudaEvent_t e = ctx->ev_pool.back();
        ctx->ev_pool.pop_back();
        return e;
    }
    cudaEvent_t e;
    cudaEventCreate(&e);
    return e;
}

struct ProfScope {
    bzk_ctx *ctx; cudaStream_t s; int kind; cudaEvent_t a = nullptr;
    ProfScope(bzk_ctx *c, cudaStream_t st, int k) : ctx(c), s(st), kind(k) {
        if (ctx->prof) { a = pool_event(ctx); cudaEventRecord(a, s); }
    }
    ~ProfScope() {
        if (ctx->prof) {
            cudaEvent_t b = pool_event(ctx);
            cudaEventRecord(b, s);
            ctx->recs.push_back({kind, a, b});
        }
    }
};

// ---------------------------------------------------------------- planning

struct Plan {
    uint32_t k, D, order;
    uint64_t B, Bw, nwaves;
    uint32_t i0;          // first tail round (k >= 1)
    uint32_t log_h0;      // pairs of the first tail round
    uint64_t N;
    size_t elem_table;    // bytes of one table set (D * N * 32)
    // per-wave workspace layout (bytes)
    size_t off_ps, off_tick, off_part, off_bufX, off_bufY, off_out, off_seed;
    size_t total;        // device workspace bytes (excluding the loader's staging slots)
    size_t stage_bytes;  // bytes of one staging slot (host tables), 0 otherwise
    uint32_t cmax;
    bool host_tables, host_outputs, need_bufX, need_bufY, bufY_alias_input;
    uint32_t given;       // BZK_F_GIVEN_CHALLENGES
    bool multi;           // given challenges, d = 1, BN254: k_multi passes (NEXT-1)
    bool dual;            // two half-batch waves on two streams, offset by one round (see enqueue_job)
    size_t wave_bytes;    // bytes of one wave's workspace region [off_ps, off_bufY end) (dual: two copies)
    uint32_t part_nv;     // field elements per CTA partial (D + 1, or 2^kMultiM column sums)
    bool gl;              // BZK_F_FIELD_GOLDILOCKS (NEXT-2)
    size_t esz;           // bytes per element: 32 (BN254) or 8 (Goldilocks)
    size_t out_bytes_per_proof;
};

// tuning knobs (environment, read once): BZK_PPT_MAX (max pairs per thread), BZK_CTA_WAVES
// (target CTA waves per launch).  (Round 1's L2 bulk prefetch option was removed in round 2: the TMA
// staging replaced it for d >= 3, the only degree it had helped.)
struct Knobs {
    uint64_t ppt_max = 256, waves = 4;   // ppt_max sweep 32..1024: 256 best for c2, c3, m0
    // BZK_CLUSTER=N: CTAs of a proof form thread-block clusters of up to N (2, 4, 8) that combine
    // their partial sums through DSMEM.  Off by default: measured 10 % slower on B200.
    uint32_t cluster = 1;
    // k_round stages its operands into shared memory with TMA (sumcheck.cuh) instead of loading them
    // straight to registers: by default for the fused rounds of d >= 2 and round 1 of d >= 3 (B200 A/B,
    // profiles/r02/r02b_*: c2 fused rounds -11 % time, c2 round 1 +7 %, c3 both -3 %, m0 (d = 1) +3 %);
    // BZK_TMA=0 / 1 forces it off / on everywhere
    int tma = -1;
    uint32_t multi_m = 3;      // BZK_MULTI_M: rounds per k_multi pass (1..3)
    // BZK_SMALL=0/1: proofs whose tables fit a cluster's shared memory run in k_small (one launch,
    // all rounds, cluster/DSMEM reduction; small.cuh)
    uint32_t small = 1;
    // BZK_CHAIN_CHUNKS: proof chunks of bzk_commit_prove's module pipeline.  Default 1 (modules in
    // sequence): on B200 the modules do not overlap usefully -- each already fills the GPU, and the
    // co-running Merkle/sum-check streams evict the encoder's L2-resident source vectors (zk20: 32.1 ms
    // per step at 1 chunk, 32.6 / 33.7 / 36.0 ms at 2 / 4 / 8, profiles/r02/bench_zk20_ch*_r02m.json)
    uint32_t chain_chunks = 1;
    // BZK_DUAL=0/1: a one-wave device batch runs as two half-batch waves on two streams, the second
    // one round behind, so one wave's round-1 evaluation (IMAD-heavy) overlaps the other's fused rounds
    // (the paper's "different proofs in different rounds").  Off: every round kernel already
    // fills the 148 SMs, so the overlap measured +0.2 % (c2), +0.4 % (c3), +0.9 % (m0) -- within noise
    // (profiles/r02/bench_*_dual*_r02p.json)
    uint32_t dual = 0;
    // BZK_MULTI_TC=0/1: three-round known-challenge passes over >= 2^10 entries run k_multi_tc (the
    // weighted row sums and column sums as u8 tensor-core products, multiround_tc.cuh) instead of k_multi
    uint32_t multi_tc = 1;
    // BZK_R1_TC=0/1: round 1 of d = 2 BN254 proofs runs k_round1_tc (the three product sums as u8
    // tensor-core products over the pairs, round1_tc.cuh) instead of k_round<2, ., FIRST>
    uint32_t r1tc = 1;
    // BZK_FUSED_TC=0/1: the fused rounds of d = 2 BN254 proofs run k_fused_tc (folds on the integer
    // pipe, the two evaluation sums as u8 tensor-core products, fused_tc.cuh) instead of k_round
    uint32_t fused_tc = 1;
    // BZK_D3_TC=0/1: round 1 and the fused rounds of d = 3 BN254 proofs run k_fused_tc<3, ...> (the
    // last product of every point as a u8 tensor-core sum over the pairs, fused_tc.cuh) instead of k_round
    uint32_t d3tc = 1;
    // BZK_FTC_SMALL_LOG=L: d = 2 fused rounds with h <= 2^L pairs per proof run the 2-warp k_fused_tc
    // (one CTA per proof up to 2^11 pairs, fused_tc.cuh); 0 = off
    uint32_t ftc_small_log = 12;
    // BZK_R1_SW64=0/1: LSB round 1 of k_round1_tc loads each table's pairs as 64-byte rows (a_j | b_j), one
    // TMA box per table, 64-byte swizzle; 0: a and b as separate boxes of 32-byte rows
    uint32_t r1_sw64 = 1;
    // BZK_SMALL_ROUND_LOG=L: the CUDA-core global rounds without TMA staging (k_round d = 1, k_gl_round)
    // with h <= 2^L pairs per proof run CTAs of 64 threads, one per 2048 pairs (as the 2-warp k_fused_tc);
    // 0 = off
    uint32_t small_round_log = 12;
    Knobs() {
        if (const char *e = getenv("BZK_SMALL_ROUND_LOG")) small_round_log = (uint32_t)std::max(0, atoi(e));
        if (const char *e = getenv("BZK_R1_SW64")) r1_sw64 = atoi(e) ? 1 : 0;
        if (const char *e = getenv("BZK_FTC_SMALL_LOG")) ftc_small_log = (uint32_t)std::max(0, atoi(e));
        if (const char *e = getenv("BZK_D3_TC")) d3tc = atoi(e) ? 1 : 0;
        if (const char *e = getenv("BZK_FUSED_TC")) fused_tc = atoi(e) ? 1 : 0;
        if (const char *e = getenv("BZK_R1_TC")) r1tc = atoi(e) ? 1 : 0;
        if (const char *e = getenv("BZK_MULTI_TC")) multi_tc = atoi(e) ? 1 : 0;
        if (const char *e = getenv("BZK_DUAL")) dual = atoi(e) ? 1 : 0;
        if (const char *e = getenv("BZK_CHAIN_CHUNKS")) chain_chunks = std::max(1, atoi(e));
        if (const char *e = getenv("BZK_SMALL")) small = atoi(e) ? 1 : 0;
        if (const char *e = getenv("BZK_MULTI_M")) multi_m = std::max(1, std::min(3, atoi(e)));
        if (const char *e = getenv("BZK_TMA")) tma = atoi(e) ? 1 : 0;
        if (const char *e = getenv("BZK_CLUSTER")) cluster = std::max(1, std::min(8, atoi(e)));
        if (const char *e = getenv("BZK_PPT_MAX")) ppt_max = std::max(1, atoi(e));
        if (const char *e = getenv("BZK_CTA_WAVES")) waves = std::max(1, atoi(e));
    }
    uint32_t tma_for(uint32_t d, bool first) const {
        if (tma >= 0) return (uint32_t)tma;
        return first ? (d >= 3 ? 1u : 0u) : (d >= 2 ? 1u : 0u);
    }
};
const Knobs &knobs() { static Knobs k; return k; }

uint32_t ctas_for(uint64_t h, uint64_t nb) {
    // enough CTAs to fill 148 SMs x 2 resident CTAs x `waves` waves, at most ppt_max pairs per thread
    const uint64_t target = (uint64_t)kSMs * 2 * knobs().waves;
    uint64_t ppt = (nb * h) / ((uint64_t)kRoundThreads * target);
    ppt = std::max<uint64_t>(1, std::min<uint64_t>(knobs().ppt_max, ppt));
    uint64_t c = (h + kRoundThreads * ppt - 1) / (kRoundThreads * ppt);
    c = std::max<uint64_t>(1, c);
    // CTAs of a proof form thread-block clusters of up to 8 (DSMEM reduction): make c a multiple
    // of the cluster size (a power of two below 8, a multiple of 8 above)
    if (c >= 8) c = (c + 7) / 8 * 8;
    else { uint64_t q = 1; while (q < c) q <<= 1; c = q; }
    return (uint32_t)c;
}

// CTAs per proof over every global round i < i0 (ctas_for is not monotone in h: ppt is floored).
// The partials buffer is sized with this maximum; each round indexes it with its own stride.
bool r1_use_tc(uint32_t D, uint64_t h);
uint32_t r1tc_ctas(uint64_t h, uint64_t nb);
bool ftc_use(uint32_t D, uint32_t i) {
    return (knobs().fused_tc && D == 2 && i >= 2) || (knobs().d3tc && D == 3);
}

// the 2-warp k_fused_tc for the small late d = 2 rounds: 2048 pairs (32 per warp-iteration, 32
// iterations) per CTA
bool ftc_small(uint32_t D, uint32_t i, uint64_t h) {
    return ftc_use(D, i) && D == 2 && knobs().ftc_small_log && h <= (1ull << knobs().ftc_small_log);
}

// the 64-thread CTAs of the late CUDA-core rounds (BZK_SMALL_ROUND_LOG)
constexpr uint32_t kSmallRoundThreads = 64;
bool small_round(uint32_t D, uint32_t i, uint64_t h, bool gl) {
    if (i < 2 || !knobs().small_round_log || h > (1ull << knobs().small_round_log)) return false;
    return gl || (!ftc_use(D, i) && !knobs().tma_for(D, false));
}

// CTAs per proof of global round i (h pairs): k_round1_tc / k_fused_tc (<= 32768 pairs per CTA: its
// s32 accumulator bound) / k_round
uint32_t round_ctas(uint32_t D, uint32_t i, uint64_t h, uint64_t nb, bool gl) {
    if (small_round(D, i, h, gl)) return (uint32_t)std::max<uint64_t>(1, h / 2048);
    if (gl) return ctas_for(h, nb);   // k_gl_round (Goldilocks: no tensor-core variants)
    if (i == 1 && r1_use_tc(D, h)) return r1tc_ctas(h, nb);
    if (ftc_small(D, i, h)) return (uint32_t)std::max<uint64_t>(1, h / 2048);
    uint32_t c = ctas_for(h, nb);
    if (ftc_use(D, i)) c = std::max<uint32_t>(c, (uint32_t)((h + 32767) / 32768));
    return c;
}

uint32_t max_round_ctas(uint32_t D, uint32_t k, uint32_t i0, uint64_t nb, bool gl) {
    uint32_t c = 1;
    for (uint32_t i = 1; i < i0; ++i) c = std::max(c, round_ctas(D, i, 1ull << (k - i), nb, gl));
    return c;
}

// Known-challenge multi-round passes (NEXT-1, d = 1): (K, m) per pass, K = variables left before the
// pass, m <= 3 rounds per pass, until the on-chip tail's K_t = k - i0 + 1 variables remain.
constexpr uint32_t kMultiM = 3;   // largest pass (k_multi instantiations; partials hold 2^kMultiM sums)
std::vector<std::pair<uint32_t, uint32_t>> multi_passes(uint32_t k, uint32_t i0) {
    std::vector<std::pair<uint32_t, uint32_t>> v;
    const uint32_t Kt = k - i0 + 1;
    for (uint32_t K = k; K > Kt;) {
        const uint32_t m = std::min(knobs().multi_m, K - Kt);
        v.push_back({K, m});
        K -= m;
    }
    return v;
}

// k_multi_tc for a pass of 3 rounds whose output has at least one 128-column tile
bool multi_use_tc(uint32_t K, uint32_t m) { return knobs().multi_tc && m == 3 && K >= 10; }

// k_multi_tc CTAs per proof: one resident CTA per SM, so >= 2 x 148 CTAs in all when the batch is
// small, >= 4 tiles per CTA, and <= 2^16 tiles per CTA (its TMEM column byte sums stay < 2^31)
uint32_t multi_tc_ctas(uint64_t Ny, uint64_t nb) {
    const uint64_t T = Ny / kTcTileRows;
    // BZK_TC_CTAS (tests): force the CTAs per proof, clamped to [1, tiles] (ragged tile counts per CTA)
    if (const char *e = getenv("BZK_TC_CTAS")) return (uint32_t)std::max<uint64_t>(1, std::min<uint64_t>(T, atoi(e)));
    uint64_t c = (2 * kSMs + nb - 1) / nb;
    c = std::min<uint64_t>(c, std::max<uint64_t>(1, T / 4));
    c = std::max<uint64_t>(c, (T + 65535) / 65536);
    return (uint32_t)c;
}

// k_round1_tc (d = 2 round 1): one resident CTA per SM, >= 2 x 148 CTAs in all when the batch is small,
// >= 8 tiles of 128 pairs per CTA, <= 2^21 pairs per CTA (its 64-bit anti-diagonal sums stay < 2^43)
bool r1_use_tc(uint32_t D, uint64_t h) { return knobs().r1tc && D == 2 && h >= 128; }
uint32_t r1tc_ctas(uint64_t h, uint64_t nb) {
    const uint64_t T = h / 128;
    // BZK_R1TC_CTAS (tests): force the CTAs per proof, clamped to [1, tiles] (ragged tile counts per CTA)
    if (const char *e = getenv("BZK_R1TC_CTAS")) return (uint32_t)std::max<uint64_t>(1, std::min<uint64_t>(T, atoi(e)));
    uint64_t c = (2 * kSMs + nb - 1) / nb;
    c = std::min<uint64_t>(c, std::max<uint64_t>(1, T / 8));
    c = std::max<uint64_t>(c, (h + (1ull << 21) - 1) >> 21);
    return (uint32_t)c;
}

uint32_t multi_pass_ctas(uint32_t K, uint32_t m, uint64_t nb) {
    return multi_use_tc(K, m) ? multi_tc_ctas(1ull << (K - m), nb) : ctas_for(1ull << (K - m), nb);
}

uint32_t max_multi_ctas(uint32_t k, uint32_t i0, uint64_t nb) {
    uint32_t c = 1;
    for (auto &pm : multi_passes(k, i0)) c = std::max(c, multi_pass_ctas(pm.first, pm.second, nb));
    return c;
}

uint32_t cluster_for(uint32_t ctas) {
    uint32_t c = 1;
    while (c * 2 <= knobs().cluster && ctas % (c * 2) == 0) c *= 2;
    return c;
}

size_t align_up(size_t x) { return (x + 255) & ~(size_t)255; }

bzk_status validate_args(bzk_ctx *ctx, const bzk_batch *b) {
    if (!b) return fail(ctx, BZK_EINVAL, "batch is NULL");
    if (b->num_vars > 30) return fail(ctx, BZK_EINVAL, "num_vars must be <= 30");
    if (b->degree < 1) return fail(ctx, BZK_EINVAL, "degree must be >= 1");
    if (b->degree > 4) return fail(ctx, BZK_EUNSUPPORTED, "degree > 4 is not built (kernels exist for d = 1..4)");
    if (b->order > 1) return fail(ctx, BZK_EINVAL, "order must be BZK_ORDER_LSB or BZK_ORDER_MSB");
    if (b->batch == 0) return fail(ctx, BZK_EINVAL, "batch must be >= 1");
    if (!b->seed) return fail(ctx, BZK_EINVAL, "seed is NULL");
    if (!b->tables) return fail(ctx, BZK_EINVAL, "tables is NULL");
    if (b->num_vars > 0 && (!b->round_evals || !b->challenges))
        return fail(ctx, BZK_EINVAL, "round_evals/challenges is NULL");
    if (!b->final_evals) return fail(ctx, BZK_EINVAL, "final_evals is NULL");
    if (b->tables_mem > 1 || b->outputs_mem > 1) return fail(ctx, BZK_EINVAL, "bad *_mem value");
    if (b->batch - 1 > ~0ull - b->first_index) return fail(ctx, BZK_EINVAL, "first_index + batch exceeds 2^64");
    // BN254 kernels access elements with 256-bit loads/stores: device buffers must be 32-byte aligned
    if (!(b->flags & BZK_F_FIELD_GOLDILOCKS)) {
        auto mis = [](const void *q) { return q && ((uintptr_t)q & 31u); };
        if (b->tables_mem == BZK_MEM_DEVICE && mis(b->tables))
            return fail(ctx, BZK_EINVAL, "device tables must be 32-byte aligned");
        if (b->outputs_mem == BZK_MEM_DEVICE &&
            (mis(b->round_evals) || mis(b->challenges) || mis(b->final_evals) || mis(b->claims)))
            return fail(ctx, BZK_EINVAL, "device outputs must be 32-byte aligned");
    }
    return BZK_OK;
}

int small_cs_log(uint32_t D, uint32_t k, uint64_t nb);   // k_small eligibility (run_wave)

bzk_status make_plan(bzk_ctx *ctx, const bzk_batch *b, Plan &P) {
    P.k = b->num_vars; P.D = b->degree; P.order = b->order; P.B = b->batch;
    P.N = 1ull << P.k;
    P.gl = (b->flags & BZK_F_FIELD_GOLDILOCKS) != 0;
    P.esz = P.gl ? 8 : 32;
    P.elem_table = (size_t)P.D * P.N * P.esz;
    P.host_tables = b->tables_mem == BZK_MEM_HOST;
    P.host_outputs = b->outputs_mem == BZK_MEM_HOST;
    P.given = (b->flags & BZK_F_GIVEN_CHALLENGES) ? 1u : 0u;
    if (P.k == 0) { P.i0 = 1; P.log_h0 = 0; }
    else if (P.k - 1 <= kTailLog) { P.i0 = 1; P.log_h0 = P.k - 1; }
    else { P.i0 = P.k - kTailLog; P.log_h0 = kTailLog; }
    // given challenges, d = 1 (Alg. 1): k_multi passes, several rounds per read of the table (NEXT-1)
    P.multi = P.given && P.D == 1 && !P.gl && P.i0 > 1;
    P.part_nv = P.multi ? (1u << kMultiM) : P.D + 1;
    const bool preserve = (b->flags & BZK_F_PRESERVE_INPUT) != 0;
    P.need_bufX = P.i0 > 2;
    P.need_bufY = P.i0 > 3;
    // consume mode (or host tables staged into our own buffers): round 3+ may overwrite the input
    P.bufY_alias_input = P.need_bufY && (P.host_tables || !preserve);
    P.out_bytes_per_proof = P.esz * ((size_t)P.k * (P.D + 1) + P.k + P.D + 1);

    size_t limit = ctx->workspace_limit;
    if (limit == 0) {
        // free device memory + our own reusable allocations - 2 GiB; cached until we (re)allocate
        if (ctx->auto_limit == 0) {
            size_t fr = 0, tot = 0;
            cudaMemGetInfo(&fr, &tot);
            fr += ctx->ws_size + 2 * ctx->stage_size;
            ctx->auto_limit = fr > (2ull << 30) ? fr - (2ull << 30) : fr / 2;
        }
        limit = ctx->auto_limit;
    }
    auto per_proof = [&](uint64_t bw) -> size_t {
        (void)bw;
        size_t s = std::max(sizeof(ProofState), sizeof(gl::State)) + 4;
        uint32_t c = P.k ? (P.multi ? max_multi_ctas(P.k, P.i0, bw) : max_round_ctas(P.D, P.k, P.i0, bw, P.gl)) : 1;
        s += (size_t)c * P.part_nv * P.esz;
        if (P.need_bufX) s += (size_t)P.D * (P.N / 2) * P.esz;
        if (P.need_bufY && !P.bufY_alias_input) s += (size_t)P.D * (P.N / 4) * P.esz;
        if (P.host_tables) s += 2 * P.elem_table;
        return s;
    };
    const size_t fixed = 4096 + (P.host_outputs ? align_up(P.B * P.out_bytes_per_proof) : 0);
    uint64_t bw = std::min<uint64_t>(P.B, 65535);
    // large host-table jobs: at least 8 loader waves so the H2D of wave w+1 overlaps the compute
    // of wave w (small jobs overlap with the neighbouring jobs instead)
    if (P.host_tables && P.B >= 8 && P.B * P.elem_table > (2ull << 30)) bw = std::min<uint64_t>(bw, (P.B + 7) / 8);
    while (bw > 1 && fixed + per_proof(bw) * bw + 8 * 256 > limit) bw = (bw + 1) / 2;
    if (fixed + per_proof(bw) * bw + 8 * 256 > limit)
        return fail(ctx, BZK_ENOMEM, "workspace_limit too small for one proof");
    // balance the waves
    uint64_t nw = (P.B + bw - 1) / bw;
    bw = (P.B + nw - 1) / nw;
    P.dual = knobs().dual && nw == 1 && P.B >= 2 && !P.host_tables && !P.gl && !P.multi && P.i0 > 2 &&
             small_cs_log(P.D, P.k, P.B) < 0;
    if (P.dual) { nw = 2; bw = (P.B + 1) / 2; }   // two waves of B/2: the same scratch as one wave of B
    P.Bw = bw; P.nwaves = nw;
    P.cmax = P.k ? std::max(max_round_ctas(P.D, P.k, P.i0, bw, P.gl), max_round_ctas(P.D, P.k, P.i0, P.B - (nw - 1) * bw, P.gl)) : 1;
    if (P.multi) P.cmax = std::max(max_multi_ctas(P.k, P.i0, bw), max_multi_ctas(P.k, P.i0, P.B - (nw - 1) * bw));

    size_t off = 0;
    P.off_seed = off; off += 256;
    P.off_ps = off; off = align_up(off + bw * std::max(sizeof(ProofState), sizeof(gl::State)));
    P.off_tick = off; off = align_up(off + bw * 4);
    P.off_part = off; off = align_up(off + (size_t)bw * P.cmax * P.part_nv * P.esz);
    P.off_bufX = off; if (P.need_bufX) off = align_up(off + (size_t)bw * P.D * (P.N / 2) * P.esz);
    P.off_bufY = off; if (P.need_bufY && !P.bufY_alias_input) off = align_up(off + (size_t)bw * P.D * (P.N / 4) * P.esz);
    P.wave_bytes = off - P.off_ps;
    if (P.dual) off += P.wave_bytes;              // the second wave's copy of [ps .. bufY]
    P.off_out = off; if (P.host_outputs) off = align_up(off + P.B * P.out_bytes_per_proof);
    P.total = off;
    P.stage_bytes = P.host_tables ? align_up(bw * P.elem_table) : 0;
    return BZK_OK;
}

// a cached CUDA graph holds raw workspace / staging pointers: drop it whenever they move
void drop_graph(bzk_ctx *ctx) {
    if (ctx->graph_exec) cudaGraphExecDestroy(ctx->graph_exec);
    ctx->graph_exec = nullptr;
    ctx->graph_key.clear();
    ctx->graph_launches = 0;
}

// order this call after the context's previous call (whatever stream it ran on)
bzk_status call_begin(bzk_ctx *ctx, cudaStream_t s) {
    if (ctx->ev_done_recorded) CK(cudaStreamWaitEvent(s, ctx->ev_done, 0));
    return BZK_OK;
}

bzk_status call_end(bzk_ctx *ctx, cudaStream_t s) {
    CK(cudaEventRecord(ctx->ev_done, s));
    ctx->ev_done_recorded = true;
    return BZK_OK;
}

bzk_status ensure_ws(bzk_ctx *ctx, size_t bytes) {
    if (ctx->ws_size >= bytes) return BZK_OK;
    ctx->auto_limit = 0;
    drop_graph(ctx);
    cudaDeviceSynchronize();   // earlier calls (any stream) may still use the old workspace
    if (ctx->ws) { cudaFree(ctx->ws); ctx->ws = nullptr; ctx->ws_size = 0; }
    cudaError_t e = cudaMalloc(&ctx->ws, bytes);
    if (e != cudaSuccess) {
        cudaGetLastError();
        return fail(ctx, BZK_ENOMEM, std::string("cudaMalloc workspace: ") + cudaGetErrorString(e));
    }
    ctx->ws_size = bytes;
    return BZK_OK;
}

bzk_status ensure_stage(bzk_ctx *ctx, size_t bytes) {
    if (bytes == 0 || ctx->stage_size >= bytes) return BZK_OK;
    cudaDeviceSynchronize();   // slots may still be in use by earlier work
    ctx->auto_limit = 0;
    drop_graph(ctx);
    for (int i = 0; i < 2; ++i) {
        if (ctx->stage[i]) cudaFree(ctx->stage[i]);
        ctx->stage[i] = nullptr;
    }
    ctx->stage_size = 0;
    ctx->slot_used[0] = ctx->slot_used[1] = false;
    for (int i = 0; i < 2; ++i) {
        cudaError_t e = cudaMalloc(&ctx->stage[i], bytes);
        if (e != cudaSuccess) {
            cudaGetLastError();
            return fail(ctx, BZK_ENOMEM, std::string("cudaMalloc staging: ") + cudaGetErrorString(e));
        }
    }
    ctx->stage_size = bytes;
    return BZK_OK;
}

// ---------------------------------------------------------------- kernel dispatch

cudaError_t dispatch_round(uint32_t D, uint32_t order, bool first, dim3 grid, uint32_t threads, cudaStream_t s,
                           const RoundParams &p, const CUtensorMap &tm) {
    switch (D) {
        case 1: return launch_round<1>(order, first, grid, threads, s, p, tm);
        case 2: return launch_round<2>(order, first, grid, threads, s, p, tm);
        case 3: return launch_round<3>(order, first, grid, threads, s, p, tm);
        case 4: return launch_round<4>(order, first, grid, threads, s, p, tm);
    }
    return cudaErrorInvalidValue;
}

// cuTensorMapEncodeTiled through the runtime's driver entry point (no link-time libcuda dependency)
PFN_cuTensorMapEncodeTiled_v12000 tensor_map_encoder() {
    static PFN_cuTensorMapEncodeTiled_v12000 fn = [] {
        void *p = nullptr;
        cudaDriverEntryPointQueryResult q;
        if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) != cudaSuccess ||
            q != cudaDriverEntryPointSuccess)
            p = nullptr;
        return reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(p);
    }();
    return fn;
}

// The wave's source buffer as rows of 128 B (32 x u32) with the 128-byte swizzle; boxes of box_rows
// rows (sumcheck.cuh TmaGeo).  rows = buffer bytes / 128.
bool make_row_map(CUtensorMap *tm, const void *base, uint64_t rows, uint32_t box_rows) {
    PFN_cuTensorMapEncodeTiled_v12000 enc = tensor_map_encoder();
    if (!enc) return false;
    cuuint64_t dims[2] = {32, rows};
    cuuint64_t strides[1] = {128};
    cuuint32_t box[2] = {32, box_rows};
    cuuint32_t estr[2] = {1, 1};
    return enc(tm, CU_TENSOR_MAP_DATA_TYPE_UINT32, 2, const_cast<void *>(base), dims, strides, box, estr,
               CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
               CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

// k_multi_tc's tile map (multiround_tc.cuh): 32-byte rows (8 u32), 32-byte swizzle, 128 rows per box.
// MSB: dims (8, Ny, 8 segments, B), one box = all 8 segments of a tile; LSB: dims (8, 8 entries of a
// column, Ny, B), one box per segment.
// k_round1_tc's map over the wave's round-1 tables ([tables][2h] entries of 32 bytes): 32-byte rows,
// 32-byte swizzle, 128 pairs per box.  MSB (a = j, b = j + h): dims (8, h, 2, tables), one box holds
// a table's a and b tiles; LSB (a = 2j, b = 2j + 1): dims (8, 2, h, tables), one box per tile.
bool make_r1_map(CUtensorMap *tm, uint32_t order, const void *base, uint64_t h, uint64_t tables) {
    PFN_cuTensorMapEncodeTiled_v12000 enc = tensor_map_encoder();
    if (!enc) return false;
    if (order == 0 && knobs().r1_sw64) {   // rows (a_j | b_j) of 64 bytes: dims (16 w, h, tables)
        cuuint64_t dims3[3] = {16, h, tables}, strides3[2] = {64, 2 * h * 32};
        cuuint32_t box3[3] = {16, 128, 1}, estr3[3] = {1, 1, 1};
        return enc(tm, CU_TENSOR_MAP_DATA_TYPE_UINT32, 3, const_cast<void *>(base), dims3, strides3, box3, estr3,
                   CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_64B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                   CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
    }
    cuuint64_t dims[4], strides[3];
    cuuint32_t box[4], estr[4] = {1, 1, 1, 1};
    if (order == 1) {
        dims[0] = 8; dims[1] = h; dims[2] = 2; dims[3] = tables;
        strides[0] = 32; strides[1] = h * 32; strides[2] = 2 * h * 32;
        box[0] = 8; box[1] = 128; box[2] = 2; box[3] = 1;
    } else {
        dims[0] = 8; dims[1] = 2; dims[2] = h; dims[3] = tables;
        strides[0] = 32; strides[1] = 64; strides[2] = 2 * h * 32;
        box[0] = 8; box[1] = 1; box[2] = 128; box[3] = 1;
    }
    return enc(tm, CU_TENSOR_MAP_DATA_TYPE_UINT32, 4, const_cast<void *>(base), dims, strides, box, estr,
               CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_32B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
               CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

bool make_multi_tc_map(CUtensorMap *tm, uint32_t order, const void *base, uint64_t Ny, uint64_t stride,
                       uint64_t nb) {
    PFN_cuTensorMapEncodeTiled_v12000 enc = tensor_map_encoder();
    if (!enc) return false;
    cuuint64_t dims[4], strides[3];
    cuuint32_t box[4], estr[4] = {1, 1, 1, 1};
    if (order == 1) {
        dims[0] = 8; dims[1] = Ny; dims[2] = 8; dims[3] = nb;
        strides[0] = 32; strides[1] = Ny * 32; strides[2] = stride * 32;
        box[0] = 8; box[1] = kTcTileRows; box[2] = 8; box[3] = 1;
    } else {
        dims[0] = 8; dims[1] = 8; dims[2] = Ny; dims[3] = nb;
        strides[0] = 32; strides[1] = 256; strides[2] = stride * 32;
        box[0] = 8; box[1] = 1; box[2] = kTcTileRows; box[3] = 1;
    }
    return enc(tm, CU_TENSOR_MAP_DATA_TYPE_UINT32, 4, const_cast<void *>(base), dims, strides, box, estr,
               CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_32B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
               CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

cudaError_t dispatch_tail(uint32_t D, uint32_t order, uint32_t grid, size_t smem, cudaStream_t s,
                          const TailParams &p) {
    switch (D) {
        case 1: return launch_tail<1>(order, grid, kThreads, smem, s, p);
        case 2: return launch_tail<2>(order, grid, kThreads, smem, s, p);
        case 3: return launch_tail<3>(order, grid, kThreads, smem, s, p);
        case 4: return launch_tail<4>(order, grid, kThreads, smem, s, p);
    }
    return cudaErrorInvalidValue;
}

__global__ void k_validate_gl(const uint64_t *t, uint64_t n, uint32_t *flag) {
    for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x)
        if (t[i] >= gl::P) atomicOr(flag, 1u);
}

__global__ void k_validate(const fe *t, uint64_t n, uint32_t *flag) {
    for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n;
         i += (uint64_t)gridDim.x * blockDim.x) {
        fe v = ld_fe(t + i);
        if (!fe_is_canon(v)) atomicOr(flag, 1u);
    }
}

// ---------------------------------------------------------------- one wave

struct WaveIO {
    char *ws;          // this wave's workspace base (ctx->ws, or + wave_bytes for the second dual wave)
    cudaEvent_t ev_r1; // if set: recorded on the wave's stream right after its round-1 launch (dual)
    Seed32 seed;       // transcript seed, passed to the kernel by value
    const uint8_t *seeds;   // BZK_F_SEEDS_DEVICE: this wave's per-proof seeds (device [nb][32]), else null
    char *tables;      // device tables of this wave [nb][D][N] x esz
    char *round_evals, *challenges, *final_evals, *claims;   // device outputs of this wave
    uint64_t nb, first_index;
};

// Goldilocks wave (gl.cuh): same schedule as run_wave, 8-byte elements
bzk_status run_wave_gl(bzk_ctx *ctx, const Plan &P, const WaveIO &io, cudaStream_t s) {
    char *ws = io.ws;
    gl::State *ps = (gl::State *)(ws + P.off_ps);
    uint32_t *tick = (uint32_t *)(ws + P.off_tick);
    uint64_t *part = (uint64_t *)(ws + P.off_part);
    uint64_t *tab = (uint64_t *)io.tables;
    uint64_t *bufX = (uint64_t *)(ws + P.off_bufX);
    uint64_t *bufY = P.bufY_alias_input ? tab : (uint64_t *)(ws + P.off_bufY);
    const uint32_t D = P.D, k = P.k;
    {
        ProfScope ps_(ctx, s, 3);
        cudaError_t e = gl_launch_init(ps, (uint32_t)io.nb, io.seed.b, io.seeds, io.first_index, k, D, P.order, s);
        ++ctx->launches;
        if (e != cudaSuccess) return cuda_fail(ctx, e, "gl init launch");
    }
    for (uint32_t i = 1; i < P.i0; ++i) {
        gl::RoundParams rp;
        memset(&rp, 0, sizeof rp);
        rp.log_h = k - i; rp.round = i; rp.k = k; rp.order = P.order; rp.given = P.given;
        rp.ctas = round_ctas(D, i, 1ull << rp.log_h, io.nb, true);   // the partials are sized with the same count
        rp.partials = part; rp.tickets = tick; rp.ps = ps;
        rp.round_evals = (uint64_t *)io.round_evals; rp.challenges = (uint64_t *)io.challenges;
        rp.claims = (uint64_t *)io.claims;
        if (i == 1) { rp.src = tab; rp.dst = nullptr; }
        else {
            rp.src = (i == 2) ? tab : ((i - 1) % 2 == 0 ? bufX : bufY);
            rp.dst = (i % 2 == 0) ? bufX : bufY;
        }
        if (rp.ctas > P.cmax)   // the per-CTA partials are sized for P.cmax CTAs per proof (round_ctas)
            return fail(ctx, BZK_ECUDA, "internal: round CTA count above the partials' sizing");
        dim3 grid(rp.ctas, (uint32_t)io.nb);
        ProfScope ps_(ctx, s, i == 1 ? 0 : 1);
        cudaError_t e = gl_launch_round(D, P.order, i == 1, grid,
                                        small_round(D, i, 1ull << rp.log_h, true) ? kSmallRoundThreads : kThreads, s, rp);
        ++ctx->launches;
        if (e != cudaSuccess) return cuda_fail(ctx, e, "k_gl_round launch");
    }
    {
        gl::TailParams tp;
        memset(&tp, 0, sizeof tp);
        tp.i0 = P.i0; tp.log_h0 = P.log_h0; tp.k = k; tp.order = P.order; tp.ps = ps; tp.given = P.given;
        tp.round_evals = (uint64_t *)io.round_evals; tp.challenges = (uint64_t *)io.challenges;
        tp.final_evals = (uint64_t *)io.final_evals; tp.claims = (uint64_t *)io.claims;
        tp.src = (P.i0 <= 2) ? tab : (((P.i0 - 1) % 2 == 0) ? bufX : bufY);
        size_t smem = k == 0 ? 0 : (size_t)D * 3 * (1ull << P.log_h0) * 8;
        ProfScope ps_(ctx, s, 2);
        cudaError_t e = gl_launch_tail(D, P.order, (uint32_t)io.nb, kThreads, smem, s, tp);
        ++ctx->launches;
        if (e != cudaSuccess) return cuda_fail(ctx, e, "k_gl_tail launch");
    }
    return BZK_OK;
}

// cluster size (log2) of k_small for this shape, or -1: the smallest cluster whose CTAs hold their share
// of the tables in <= kSmallSmem bytes, widened (up to 8 CTAs) while the batch leaves SMs idle.  Only
// for batches that do not fill the GPU (fewer clusters than SMs): k_small is the LATENCY path -- a
// cluster idles while its leader hashes, which lockstep per-round kernels amortise over many proofs
// (B200 A/B, profiles/r02/r02h_*: c1 0.207 -> see DESIGN sec. 8; c4's jobs 2.2x slower in k_small)
constexpr size_t kSmallSmem = 200 * 1024;
int small_cs_log(uint32_t D, uint32_t k, uint64_t nb) {
    if (k == 0 || !knobs().small) return -1;
    int c = -1;
    for (int cl = 0; cl <= 3 && cl <= (int)k; ++cl)
        if ((size_t)D * (((size_t)1 << k) >> cl) * 3 / 2 * sizeof(fe) <= kSmallSmem) { c = cl; break; }
    if (c < 0 || nb * (1ull << c) > kSMs) return -1;
    while (c < 3 && c < (int)k && nb * (2ull << c) <= (uint64_t)2 * kSMs) ++c;   // latency: spread small batches
    return c;
}

bzk_status run_wave_small(bzk_ctx *ctx, const Plan &P, const WaveIO &io, cudaStream_t s, int cs_log) {
    SmallParams sp;
    memset(&sp, 0, sizeof sp);
    sp.src = (const fe *)io.tables; sp.k = P.k; sp.cs_log = (uint32_t)cs_log; sp.order = P.order; sp.given = P.given;
    sp.first_index = io.first_index; sp.seed = io.seed; sp.seeds = io.seeds;
    sp.ps = (ProofState *)(io.ws + P.off_ps);
    sp.round_evals = (fe *)io.round_evals; sp.challenges = (fe *)io.challenges; sp.final_evals = (fe *)io.final_evals;
    sp.claims = (fe *)io.claims;
    const uint32_t cs = 1u << cs_log;
    const size_t smem = (size_t)P.D * ((P.N >> cs_log)) * 3 / 2 * sizeof(fe);
    dim3 grid(cs, (uint32_t)io.nb);
    cudaError_t e = cudaSuccess;
    {
        ProfScope ps_(ctx, s, 10);
        switch (P.D) {
            case 1: e = launch_small<1>(P.order, grid, cs, smem, s, sp); break;
            case 2: e = launch_small<2>(P.order, grid, cs, smem, s, sp); break;
            case 3: e = launch_small<3>(P.order, grid, cs, smem, s, sp); break;
            case 4: e = launch_small<4>(P.order, grid, cs, smem, s, sp); break;
        }
    }
    ++ctx->launches;
    if (e != cudaSuccess) return cuda_fail(ctx, e, "k_small launch");
    return BZK_OK;
}

bzk_status run_wave(bzk_ctx *ctx, const Plan &P, const WaveIO &io, cudaStream_t s) {
    NvtxRange nv_("bzk wave");
    {
        const int cs_log = small_cs_log(P.D, P.k, io.nb);
        if (cs_log >= 0) return run_wave_small(ctx, P, io, s, cs_log);
    }
    char *ws = io.ws;
    ProofState *ps = (ProofState *)(ws + P.off_ps);
    uint32_t *tick = (uint32_t *)(ws + P.off_tick);
    fe *part = (fe *)(ws + P.off_part);
    fe *bufX = (fe *)(ws + P.off_bufX);
    fe *tab = (fe *)io.tables;
    fe *bufY = P.bufY_alias_input ? tab : (fe *)(ws + P.off_bufY);
    const uint32_t D = P.D, k = P.k;
    {
        ProfScope ps_(ctx, s, 3);
        k_transcript_init<<<(uint32_t)((io.nb + 127) / 128), 128, 0, s>>>(ps, (uint32_t)io.nb, io.seed, io.seeds,
                                                                          io.first_index, k, D, P.order);
        ++ctx->launches;
        CK(cudaGetLastError());
    }
    const fe *tail_src = nullptr;       // multi passes: the folded round-i0 table for k_tail
    uint64_t tail_stride = 0;
    if (P.multi) {
        // NEXT-1: m rounds per read of the table (multiround.cuh).  MSB folds in place after the first
        // pass (each thread owns its column); LSB ping-pongs between the two scratch buffers.
        const fe *cur = tab;
        uint64_t cur_stride = P.N;
        uint32_t round = 1;
        for (auto &pm : multi_passes(k, P.i0)) {
            const uint32_t K = pm.first, m = pm.second;
            MultiParams mp;
            memset(&mp, 0, sizeof mp);
            mp.src = cur; mp.src_stride = cur_stride;
            if (round == 1) { mp.dst = bufX; mp.dst_stride = 1ull << (K - m); }
            else if (P.order == 1) { mp.dst = const_cast<fe *>(cur); mp.dst_stride = cur_stride; }
            else { mp.dst = (cur == bufX) ? bufY : bufX; mp.dst_stride = 1ull << (K - m); }
            mp.logK = K; mp.round0 = round; mp.k = k;
            const bool use_tc = multi_use_tc(K, m);
            mp.ctas = multi_pass_ctas(K, m, io.nb);
            mp.partials = part; mp.tickets = tick;
            mp.challenges = (const fe *)io.challenges; mp.round_evals = (fe *)io.round_evals;
            mp.claims = (fe *)io.claims;
            dim3 grid(mp.ctas, (uint32_t)io.nb);
            CUtensorMap tm;
            memset(&tm, 0, sizeof tm);
            const bool tma = !use_tc && P.order == 1 && knobs().tma != 0;   // MSB: segment-wise TMA staging
            if (tma && !make_row_map(&tm, mp.src, io.nb * cur_stride / 4, 8))
                return fail(ctx, BZK_ECUDA, "cuTensorMapEncodeTiled failed (k_multi)");
            if (use_tc && !make_multi_tc_map(&tm, P.order, mp.src, 1ull << (K - m), cur_stride, io.nb))
                return fail(ctx, BZK_ECUDA, "cuTensorMapEncodeTiled failed (k_multi_tc)");
            ProfScope ps_(ctx, s, use_tc ? 11 : 9);
            cudaError_t e = use_tc ? multi_tc_launch(P.order, grid, s, mp, tm) : multi_launch(P.order, m, tma, grid, s, mp, tm);
            ++ctx->launches;
            if (e != cudaSuccess) return cuda_fail(ctx, e, "k_multi launch");
            cur = mp.dst; cur_stride = mp.dst_stride;
            round += m;
        }
        tail_src = cur;
        tail_stride = cur_stride;
    }
    for (uint32_t i = 1; i < (P.multi ? 1u : P.i0); ++i) {
        RoundParams rp;
        memset(&rp, 0, sizeof rp);
        rp.log_h = k - i;
        rp.round = i; rp.k = k; rp.order = P.order;
        const uint64_t h = 1ull << rp.log_h;
        rp.ctas = round_ctas(D, i, h, io.nb, false);
        rp.partials = part; rp.tickets = tick; rp.ps = ps;
        rp.round_evals = (fe *)io.round_evals; rp.challenges = (fe *)io.challenges; rp.claims = (fe *)io.claims;
        rp.consts = ctx->consts;
        rp.given = P.given;
        rp.cluster = cluster_for(rp.ctas);
        if (i == 1) { rp.src = tab; rp.dst = nullptr; }
        else {
            rp.src = (i == 2) ? tab : ((i - 1) % 2 == 0 ? bufX : bufY);
            rp.dst = (i % 2 == 0) ? bufX : bufY;
        }
        CUtensorMap tm;
        memset(&tm, 0, sizeof tm);
        const bool r1tc = i == 1 && r1_use_tc(D, h), ftc = ftc_use(D, i);
        if (r1tc || ftc) {
            rp.ctas = round_ctas(D, i, h, io.nb, false);
            rp.cluster = 1;
        }
        if (r1tc && !make_r1_map(&tm, P.order, tab, h, io.nb * D))
            return fail(ctx, BZK_ECUDA, "cuTensorMapEncodeTiled failed (k_round1_tc)");
        rp.tma = r1tc ? 0 : ftc ? 1 : knobs().tma_for(D, i == 1);
        if (rp.tma) {
            const uint64_t E = i == 1 ? 2 : 4;   // raw entries per pair and table
            const uint32_t box = P.order == 0 ? (uint32_t)(E * 8) : 8u;
            if (!make_row_map(&tm, rp.src, io.nb * D * E * h / 4, box))
                return fail(ctx, BZK_ECUDA, "cuTensorMapEncodeTiled failed (TMA staging)");
        }
        if (rp.ctas > P.cmax)   // the per-CTA partials are sized for P.cmax CTAs per proof (round_ctas)
            return fail(ctx, BZK_ECUDA, "internal: round CTA count above the partials' sizing");
        dim3 grid(rp.ctas, (uint32_t)io.nb);
        {
            ProfScope ps_(ctx, s, i == 1 ? 0 : 1);
            cudaError_t e = r1tc  ? r1tc_launch(P.order, P.order == 0 && knobs().r1_sw64, grid, s, rp, tm)
                            : ftc ? ftc_launch(D, i == 1, ftc_small(D, i, h), P.order, grid, s, rp, tm)
                                  : dispatch_round(D, P.order, i == 1, grid,
                                                   small_round(D, i, h, false) ? kSmallRoundThreads : kRoundThreads,
                                                   s, rp, tm);
            ++ctx->launches;
            if (e != cudaSuccess) return cuda_fail(ctx, e, "k_round launch");
        }
        if (i == 1 && io.ev_r1) CK(cudaEventRecord(io.ev_r1, s));
    }
    {
        TailParams tp;
        memset(&tp, 0, sizeof tp);
        tp.i0 = P.i0; tp.log_h0 = P.log_h0; tp.k = k; tp.order = P.order; tp.ps = ps;
        tp.round_evals = (fe *)io.round_evals; tp.challenges = (fe *)io.challenges;
        tp.final_evals = (fe *)io.final_evals; tp.claims = (fe *)io.claims;
        tp.consts = ctx->consts;
        tp.given = P.given;
        if (tail_src) { tp.src = tail_src; tp.folded = 1; tp.src_stride = tail_stride; }
        else if (P.i0 <= 2) tp.src = tab;
        else tp.src = ((P.i0 - 1) % 2 == 0) ? bufX : bufY;
        size_t smem = k == 0 ? 0 : (size_t)D * 3 * (1ull << P.log_h0) * 32;
        ProfScope ps_(ctx, s, 2);
        cudaError_t e = dispatch_tail(D, P.order, (uint32_t)io.nb, smem, s, tp);
        ++ctx->launches;
        if (e != cudaSuccess) return cuda_fail(ctx, e, "k_tail launch");
    }
    return BZK_OK;
}

// Enqueue one job (all its waves) on stream s.  Host tables go through the loader ring: wave w's
// tables are copied into the next staging slot on the copy stream as soon as that slot's
// previous user (possibly a wave of the previous job or call) has been consumed, so copies run
// ahead of compute across waves AND jobs.  Returns after enqueueing (no synchronisation) unless
// validation is requested.
bzk_status enqueue_job(bzk_ctx *ctx, const bzk_batch *b, const Plan &P, cudaStream_t s) {
    NvtxRange nv_("bzk job");
    char *ws = (char *)ctx->ws;
    CK(cudaMemsetAsync(ws + P.off_tick, 0, P.Bw * 4, s));
    // dual: wave 1 runs on the context's second stream, one round behind wave 0 (its first launch waits
    // for wave 0's round-1 kernel), in its own copy of the wave workspace
    cudaStream_t s2 = s;
    cudaEvent_t ev_r1 = nullptr;
    if (P.dual) {
        if (!ctx->dual_stream) CK(cudaStreamCreateWithFlags(&ctx->dual_stream, cudaStreamNonBlocking));
        s2 = ctx->dual_stream;
        CK(cudaMemsetAsync(ws + P.wave_bytes + P.off_tick, 0, P.Bw * 4, s));
        cudaEvent_t e0 = pool_event(ctx);
        CK(cudaEventRecord(e0, s));
        CK(cudaStreamWaitEvent(s2, e0, 0));
        ctx->ev_pool.push_back(e0);
        ev_r1 = pool_event(ctx);
    }
    const bool validate = (b->flags & BZK_F_VALIDATE) != 0;
    if (validate) CK(cudaMemsetAsync(ctx->d_flag, 0, 4, s));

    const size_t E = P.esz;
    const size_t ev_pp = (size_t)P.k * (P.D + 1) * E, ch_pp = P.k * E, fi_pp = P.D * E;   // bytes per proof
    char *o_ev, *o_ch, *o_fi, *o_cl;
    if (P.host_outputs) {
        char *base = ws + P.off_out;
        o_ev = base; o_ch = o_ev + P.B * ev_pp; o_fi = o_ch + P.B * ch_pp; o_cl = o_fi + P.B * fi_pp;
        if (P.given && P.k)
            CK(cudaMemcpyAsync(o_ch, b->challenges, P.B * ch_pp, cudaMemcpyHostToDevice, s));
    } else {
        o_ev = (char *)b->round_evals; o_ch = (char *)b->challenges; o_fi = (char *)b->final_evals;
        o_cl = (char *)b->claims;
    }
    for (uint64_t w = 0; w < P.nwaves; ++w) {
        WaveIO io;
        const uint64_t b0 = w * P.Bw;
        io.ws = ws + (P.dual && w == 1 ? P.wave_bytes : 0);
        io.ev_r1 = (P.dual && w == 0) ? ev_r1 : nullptr;
        cudaStream_t sw = s;
        if (P.dual && w == 1) {
            CK(cudaStreamWaitEvent(s2, ev_r1, 0));
            sw = s2;
        }
        if (b->flags & BZK_F_SEEDS_DEVICE) {
            memset(io.seed.b, 0, 32);
            io.seeds = b->seed + b0 * 32;
        } else {
            memcpy(io.seed.b, b->seed, 32);
            io.seeds = nullptr;
        }
        io.nb = std::min<uint64_t>(P.Bw, P.B - b0);
        io.first_index = b->first_index + b0;
        io.round_evals = o_ev + b0 * ev_pp;
        io.challenges = o_ch + b0 * ch_pp;
        io.final_evals = o_fi + b0 * fi_pp;   // (byte offsets)
        io.claims = (P.host_outputs || o_cl) ? o_cl + b0 * E : nullptr;
        int slot = -1;
        if (P.host_tables) {
            slot = ctx->next_slot;
            ctx->next_slot ^= 1;
            if (ctx->slot_used[slot]) CK(cudaStreamWaitEvent(ctx->copy_stream, ctx->ev_consumed[slot], 0));
            {
                ProfScope ps_(ctx, ctx->copy_stream, 5);
                CK(cudaMemcpyAsync(ctx->stage[slot], (const char *)b->tables + b0 * P.elem_table,
                                   io.nb * P.elem_table, cudaMemcpyHostToDevice, ctx->copy_stream));
            }
            CK(cudaEventRecord(ctx->ev_copied[slot], ctx->copy_stream));
            CK(cudaStreamWaitEvent(s, ctx->ev_copied[slot], 0));
            io.tables = (char *)ctx->stage[slot];
        } else {
            io.tables = (char *)b->tables + b0 * P.elem_table;
        }
        if (validate) {
            ProfScope ps_(ctx, sw, 4);
            if (P.gl) k_validate_gl<<<kSMs * 8, 256, 0, sw>>>((const uint64_t *)io.tables, io.nb * P.D * P.N, ctx->d_flag);
            else      k_validate<<<kSMs * 8, 256, 0, sw>>>((const fe *)io.tables, io.nb * P.D * P.N, ctx->d_flag);
            ++ctx->launches;
            CK(cudaGetLastError());
        }
        bzk_status st = P.gl ? run_wave_gl(ctx, P, io, sw) : run_wave(ctx, P, io, sw);
        if (st) return st;
        if (slot >= 0) {
            CK(cudaEventRecord(ctx->ev_consumed[slot], s));
            ctx->slot_used[slot] = true;
        }
    }
    if (P.dual) {                                  // the caller's stream waits for the second wave
        cudaEvent_t e1 = pool_event(ctx);
        CK(cudaEventRecord(e1, s2));
        CK(cudaStreamWaitEvent(s, e1, 0));
        ctx->ev_pool.push_back(e1);
        ctx->ev_pool.push_back(ev_r1);
    }
    if (P.host_outputs) {
        if (P.k) {
            CK(cudaMemcpyAsync(b->round_evals, o_ev, P.B * ev_pp, cudaMemcpyDeviceToHost, s));
            if (!P.given) CK(cudaMemcpyAsync(b->challenges, o_ch, P.B * ch_pp, cudaMemcpyDeviceToHost, s));
        }
        CK(cudaMemcpyAsync(b->final_evals, o_fi, P.B * fi_pp, cudaMemcpyDeviceToHost, s));
        if (b->claims) CK(cudaMemcpyAsync(b->claims, o_cl, P.B * E, cudaMemcpyDeviceToHost, s));
    }
    if (validate) {
        uint32_t flag = 0;
        CK(cudaMemcpyAsync(&flag, ctx->d_flag, 4, cudaMemcpyDeviceToHost, s));
        CK(cudaStreamSynchronize(s));
        if (flag) return fail(ctx, BZK_ENONCANON, "an input element is >= p");
    }
    return BZK_OK;
}

// Plan every job, size the workspace for the largest, enqueue all of them, then synchronise
// when the caller asked for it or host memory is involved (outputs must be readable on return).
bzk_status prove_jobs(bzk_ctx *ctx, const bzk_batch *jobs, size_t njobs, cudaStream_t s) {
    NvtxRange nv_("bzk_prove");
    std::vector<Plan> plans(njobs);
    size_t ws_need = 0, stage_need = 0;
    bool need_sync = false;
    for (size_t j = 0; j < njobs; ++j) {
        bzk_status st = validate_args(ctx, &jobs[j]);
        if (st) return njobs > 1 ? fail(ctx, st, "job " + std::to_string(j) + ": " + ctx->last_error) : st;
        st = make_plan(ctx, &jobs[j], plans[j]);
        if (st) return st;
        ws_need = std::max(ws_need, plans[j].total);
        stage_need = std::max(stage_need, plans[j].stage_bytes);
        need_sync |= (jobs[j].flags & BZK_F_SYNC) || plans[j].host_outputs || plans[j].host_tables;
    }
    bool graph = !need_sync && !ctx->prof && s != nullptr;   // no capture on the legacy stream
    for (size_t j = 0; j < njobs; ++j)
        graph = graph && (jobs[j].flags & BZK_F_GRAPH) && !(jobs[j].flags & BZK_F_VALIDATE);
    std::vector<unsigned char> key;
    if (graph) {
        // identical job descriptions (pointers, sizes, seed bytes) on the same stream -> replay
        key.resize(njobs * (sizeof(bzk_batch) + 32) + sizeof(cudaStream_t));
        unsigned char *kp = key.data();
        memcpy(kp, &s, sizeof(s));
        kp += sizeof(s);
        for (size_t j = 0; j < njobs; ++j) {
            memcpy(kp, &jobs[j], sizeof(bzk_batch));
            // host seed: its bytes; device seeds (BZK_F_SEEDS_DEVICE): the pointer in the struct is the key
            if (jobs[j].flags & BZK_F_SEEDS_DEVICE) memset(kp + sizeof(bzk_batch), 0, 32);
            else memcpy(kp + sizeof(bzk_batch), jobs[j].seed, 32);
            kp += sizeof(bzk_batch) + 32;
        }
    }
    bzk_status st = ensure_ws(ctx, ws_need);
    if (st) return st;
    st = ensure_stage(ctx, stage_need);
    if (st) return st;
    st = call_begin(ctx, s);
    if (st) return st;
    if (graph && ctx->graph_exec && ctx->graph_key == key) {
        CK(cudaGraphLaunch(ctx->graph_exec, s));
        ctx->launches += ctx->graph_launches;
        return call_end(ctx, s);
    }
    if (graph) {
        if (ctx->graph_exec) { cudaGraphExecDestroy(ctx->graph_exec); ctx->graph_exec = nullptr; }
        CK(cudaStreamBeginCapture(s, cudaStreamCaptureModeThreadLocal));
    }
    const uint64_t l0 = ctx->launches;
    for (size_t j = 0; j < njobs; ++j) {
        st = enqueue_job(ctx, &jobs[j], plans[j], s);
        if (st) {
            if (graph) { cudaGraph_t g = nullptr; cudaStreamEndCapture(s, &g); if (g) cudaGraphDestroy(g); }
            else call_end(ctx, s);
            return st;
        }
    }
    if (graph) {
        cudaGraph_t g = nullptr;
        CK(cudaStreamEndCapture(s, &g));
        cudaError_t e = cudaGraphInstantiate(&ctx->graph_exec, g, 0);
        cudaGraphDestroy(g);
        if (e != cudaSuccess) { ctx->graph_exec = nullptr; return cuda_fail(ctx, e, "cudaGraphInstantiate"); }
        ctx->graph_key = key;
        ctx->graph_launches = ctx->launches - l0;
        CK(cudaGraphLaunch(ctx->graph_exec, s));
    }
    st = call_end(ctx, s);
    if (st) return st;
    if (need_sync) CK(cudaStreamSynchronize(s));
    return BZK_OK;
}


// ---------------------------------------------------------------- Merkle trees (NEXT-3)
//
// Plan: a chain of stage launches (merkle.cuh).  Stage s hashes M_s 64-byte blocks per tree (the
// input blocks for s = 0, pairs of level-(lvl0_s - 1) digests after that); each thread covers 2^lt
// blocks and produces one digest of level lvl0_s + lt.  Host blocks stream through the loader ring
// in waves (H2D on copy_stream); host node arrays stream back per wave on d2h_stream while the next
// wave computes ("dynamic loading and storing", multi-stream).

struct MkStage { uint32_t lt, lg_tpt, lvl0; };

// blocks per thread = 2^lt (BZK_MK_LT, default 3: tuned on B200)
uint32_t mk_lt_max() {
    static uint32_t v = [] {
        const char *e = getenv("BZK_MK_LT");
        return e ? (uint32_t)std::max(0, std::min(4, atoi(e))) : 3u;
    }();
    return v;
}

std::vector<MkStage> merkle_stages(uint32_t n) {
    std::vector<MkStage> v;
    uint32_t lgM = n, lvl0 = 0;
    for (;;) {
        MkStage st;
        st.lt = std::min(mk_lt_max(), lgM);
        st.lg_tpt = lgM - st.lt;
        st.lvl0 = lvl0;
        v.push_back(st);
        if (st.lg_tpt == 0) break;
        lvl0 = lvl0 + st.lt + 1;     // the next stage's leaf hashes are H(pair of thread roots)
        lgM = st.lg_tpt - 1;
    }
    return v;
}

// The stage chain of one wave of nb trees (device buffers): blocks [nb] x blk_stride bytes, node arrays
// (may be null) [nb] x nodes_stride, roots [nb][32]; scr[0..1]: inter-stage digests when nodes is null
// (nb x scratch_pt bytes each).
bzk_status merkle_chain(bzk_ctx *ctx, uint32_t hash, uint32_t n, const std::vector<MkStage> &stages,
                        const uint8_t *blocks, uint64_t blk_stride, uint8_t *nodes, uint64_t nodes_bytes,
                        uint8_t *roots, uint8_t *const scr[2], size_t scratch_pt, uint64_t nb, cudaStream_t s) {
    const bool dev_nodes = nodes != nullptr;
    const uint8_t *in = blocks;
    uint64_t in_stride = blk_stride;
    for (size_t si = 0; si < stages.size(); ++si) {
        const MkStage &g = stages[si];
        const bool last = si + 1 == stages.size();
        mk::StageParams p;
        p.in = in; p.in_stride = in_stride;
        p.nodes = nodes; p.nodes_stride = nodes_bytes;
        p.n = n; p.lvl0 = g.lvl0; p.lg_tpt = g.lg_tpt;
        p.threads = nb << g.lg_tpt;
        const uint32_t top = g.lvl0 + g.lt;      // level of the thread roots
        if (last) { p.out = roots; p.out_stride = 32; }
        else if (dev_nodes) { p.out = nullptr; p.out_stride = 0; }
        else { p.out = scr[si & 1]; p.out_stride = (uint64_t)32 << g.lg_tpt; }
        const uint32_t tpb = 256;
        const uint64_t grid = (p.threads + tpb - 1) / tpb;
        if (grid > 0x7fffffffull) return fail(ctx, BZK_EINVAL, "too many CTAs in one stage launch");
        {
            ProfScope ps_(ctx, s, 6);
            cudaError_t e = merkle_launch_stage(hash, g.lt, (uint32_t)grid, tpb, s, p);
            ++ctx->launches;
            if (e != cudaSuccess) return cuda_fail(ctx, e, "k_merkle_stage");
        }
        if (!last) {
            if (dev_nodes) {
                in = nodes + (((2ull << n) - (2ull << (n - top))) * 32);
                in_stride = nodes_bytes;
            } else {
                in = p.out;
                in_stride = p.out_stride;
            }
        }
    }
    (void)scratch_pt;
    return BZK_OK;
}

bzk_status merkle_impl(bzk_ctx *ctx, const bzk_merkle_batch *m, cudaStream_t s) {
    NvtxRange nv_("bzk_merkle");
    if (!m) return fail(ctx, BZK_EINVAL, "batch is NULL");
    if (m->log_blocks > 30) return fail(ctx, BZK_EINVAL, "log_blocks must be <= 30");
    if (m->hash > 1) return fail(ctx, BZK_EINVAL, "hash must be BZK_MERKLE_COMPRESS or BZK_MERKLE_SHA256");
    if (m->batch == 0) return fail(ctx, BZK_EINVAL, "batch must be >= 1");
    if (!m->blocks || !m->roots) return fail(ctx, BZK_EINVAL, "blocks/roots is NULL");
    if (m->blocks_mem > 1 || m->outputs_mem > 1) return fail(ctx, BZK_EINVAL, "bad *_mem value");
    auto mis = [](const void *q) { return q && ((uintptr_t)q & 31u); };
    if ((m->blocks_mem == BZK_MEM_DEVICE && mis(m->blocks)) ||
        (m->outputs_mem == BZK_MEM_DEVICE && (mis(m->roots) || mis(m->nodes))))
        return fail(ctx, BZK_EINVAL, "device buffers must be 32-byte aligned");
    const uint32_t n = m->log_blocks;
    const uint64_t N = 1ull << n, B = m->batch;
    const size_t blk_bytes = (size_t)N * 64, nodes_bytes = (size_t)(2 * N - 1) * 32;
    const bool host_in = m->blocks_mem == BZK_MEM_HOST, host_out = m->outputs_mem == BZK_MEM_HOST;
    const bool want_nodes = m->nodes != nullptr;
    const std::vector<MkStage> stages = merkle_stages(n);
    // scratch for CTA roots between stages when the node array is not kept on the device
    const bool dev_nodes = want_nodes;   // host_out stages the node array per wave on the device
    const size_t scratch_pt = dev_nodes ? 0 : (size_t)32 << stages[0].lg_tpt;

    size_t limit = ctx->workspace_limit;
    if (limit == 0) {
        if (ctx->auto_limit == 0) {
            size_t fr = 0, tot = 0;
            cudaMemGetInfo(&fr, &tot);
            fr += ctx->ws_size + 2 * ctx->stage_size;
            ctx->auto_limit = fr > (2ull << 30) ? fr - (2ull << 30) : fr / 2;
        }
        limit = ctx->auto_limit;
    }
    auto per_tree = [&]() {
        size_t t = 2 * scratch_pt;
        if (host_in) t += 2 * blk_bytes;
        if (host_out && want_nodes) t += 2 * nodes_bytes;
        return t;
    };
    const size_t fixed = 4096 + (host_out ? align_up(B * 32) : 0);
    uint64_t bw = B;
    if ((host_in || host_out) && B >= 8 && B * (blk_bytes + nodes_bytes) > (1ull << 30)) bw = (B + 7) / 8;
    while (bw > 1 && fixed + per_tree() * bw + 1024 > limit) bw = (bw + 1) / 2;
    if (fixed + per_tree() * bw + 1024 > limit) return fail(ctx, BZK_ENOMEM, "workspace_limit too small for one tree");
    const uint64_t nw = (B + bw - 1) / bw;
    bw = (B + nw - 1) / nw;

    size_t off = 0;
    const size_t off_roots = off; if (host_out) off = align_up(off + B * 32);
    const size_t off_scr = off; off = align_up(off + 2 * bw * scratch_pt);
    const size_t off_nodes = off; if (host_out && want_nodes) off = align_up(off + 2 * bw * nodes_bytes);
    bzk_status st = ensure_ws(ctx, std::max<size_t>(off, 256));
    if (st) return st;
    st = ensure_stage(ctx, host_in ? align_up(bw * blk_bytes) : 0);
    if (st) return st;
    st = call_begin(ctx, s);
    if (st) return st;
    char *ws = (char *)ctx->ws;
    uint8_t *roots_all = host_out ? (uint8_t *)(ws + off_roots) : m->roots;

    bool nslot_used[2] = {false, false};
    for (uint64_t w = 0; w < nw; ++w) {
        const uint64_t b0 = w * bw, nb = std::min<uint64_t>(bw, B - b0);
        const uint8_t *blocks;
        int slot = -1;
        if (host_in) {
            slot = ctx->next_slot;
            ctx->next_slot ^= 1;
            if (ctx->slot_used[slot]) CK(cudaStreamWaitEvent(ctx->copy_stream, ctx->ev_consumed[slot], 0));
            {
                ProfScope ps_(ctx, ctx->copy_stream, 5);
                CK(cudaMemcpyAsync(ctx->stage[slot], m->blocks + b0 * blk_bytes, nb * blk_bytes,
                                   cudaMemcpyHostToDevice, ctx->copy_stream));
            }
            CK(cudaEventRecord(ctx->ev_copied[slot], ctx->copy_stream));
            CK(cudaStreamWaitEvent(s, ctx->ev_copied[slot], 0));
            blocks = (const uint8_t *)ctx->stage[slot];
        } else {
            blocks = m->blocks + b0 * blk_bytes;
        }
        uint8_t *nodes = nullptr;
        const int ns = (int)(w & 1);
        if (want_nodes) {
            if (host_out) {
                nodes = (uint8_t *)(ws + off_nodes) + (size_t)ns * bw * nodes_bytes;
                if (nslot_used[ns]) CK(cudaStreamWaitEvent(s, ctx->ev_nodes_copied[ns], 0));
            } else {
                nodes = m->nodes + b0 * nodes_bytes;
            }
        }
        uint8_t *scr[2] = {(uint8_t *)(ws + off_scr), (uint8_t *)(ws + off_scr) + bw * scratch_pt};
        st = merkle_chain(ctx, m->hash, n, stages, blocks, blk_bytes, nodes, nodes_bytes, roots_all + b0 * 32, scr,
                          scratch_pt, nb, s);
        if (st) return st;
        if (slot >= 0) {
            CK(cudaEventRecord(ctx->ev_consumed[slot], s));
            ctx->slot_used[slot] = true;
        }
        if (want_nodes && host_out) {
            CK(cudaEventRecord(ctx->ev_nodes_ready[ns], s));
            CK(cudaStreamWaitEvent(ctx->d2h_stream, ctx->ev_nodes_ready[ns], 0));
            {
                ProfScope ps_(ctx, ctx->d2h_stream, 7);
                CK(cudaMemcpyAsync(m->nodes + b0 * nodes_bytes, nodes, nb * nodes_bytes, cudaMemcpyDeviceToHost,
                                   ctx->d2h_stream));
            }
            CK(cudaEventRecord(ctx->ev_nodes_copied[ns], ctx->d2h_stream));
            nslot_used[ns] = true;
        }
    }
    if (host_out) {
        CK(cudaMemcpyAsync(m->roots, roots_all, B * 32, cudaMemcpyDeviceToHost, s));
        CK(cudaStreamSynchronize(ctx->d2h_stream));
    }
    st = call_end(ctx, s);
    if (st) return st;
    if (host_in || host_out || (m->flags & BZK_F_SYNC)) CK(cudaStreamSynchronize(s));
    return BZK_OK;
}


// ---------------------------------------------------------------- linear-time encoder (NEXT-4)
//
// bzk_encoder_create converts every CSR graph to SELL-32 on the host (rows sorted by length, the
// paper's bucket sort of P:191, 32 rows per warp slice, entries lane-interleaved), uploads it in one
// allocation and turns the weights into Montgomery form on the device.  bzk_encode then runs the
// two launch chains of encoder.cuh in place on the codeword buffer.

struct SellDev {
    uint32_t rows = 0, cols = 0, slices = 0;
    uint64_t entries = 0;
    uint32_t *perm = nullptr, *slice_w = nullptr, *col = nullptr;
    uint64_t *slice_off = nullptr;
    fe *val = nullptr;
};

}  // namespace

struct bzk_encoder {
    int device = 0;
    uint32_t log_n = 0, levels = 0, m = 0;
    std::vector<SellDev> A, B;
    SellDev G0;
    void *mem = nullptr;
    size_t bytes = 0;
};

namespace {

struct SellHost {
    std::vector<uint32_t> perm, slice_w, col;
    std::vector<uint64_t> slice_off;
    std::vector<uint64_t> val;   // 4 words per entry
};

bzk_status sell_build(bzk_ctx *ctx, const bzk_csr &M, SellHost &H, std::string &why) {
    if (!M.row_ptr || !M.col || !M.val) { why = "CSR pointer is NULL"; return BZK_EINVAL; }
    const uint32_t rows = M.rows;
    std::vector<uint32_t> len(rows);
    for (uint32_t r = 0; r < rows; ++r) {
        if (M.row_ptr[r + 1] < M.row_ptr[r]) { why = "row_ptr not monotone"; return BZK_EINVAL; }
        len[r] = M.row_ptr[r + 1] - M.row_ptr[r];
    }
    if (M.row_ptr[rows] != M.nnz) { why = "row_ptr[rows] != nnz"; return BZK_EINVAL; }
    for (uint64_t e = 0; e < M.nnz; ++e)
        if (M.col[e] >= M.cols) { why = "column index out of range"; return BZK_EINVAL; }
    // bucket sort of the rows by length, longest first
    const uint32_t maxlen = rows ? *std::max_element(len.begin(), len.end()) : 0;
    std::vector<uint32_t> cnt(maxlen + 2, 0);
    for (uint32_t r = 0; r < rows; ++r) ++cnt[maxlen - len[r]];
    std::vector<uint32_t> start(maxlen + 2, 0);
    for (uint32_t k = 1; k <= maxlen + 1; ++k) start[k] = start[k - 1] + cnt[k - 1];
    std::vector<uint32_t> order(rows);
    for (uint32_t r = 0; r < rows; ++r) order[start[maxlen - len[r]]++] = r;
    const uint32_t slices = (rows + 31) / 32;
    H.perm.assign((size_t)slices * 32, 0xffffffffu);
    H.slice_w.assign(slices, 0);
    H.slice_off.assign(slices, 0);
    uint64_t total = 0;
    for (uint32_t sl = 0; sl < slices; ++sl) {
        H.slice_w[sl] = len[order[(size_t)sl * 32]];
        H.slice_off[sl] = total;
        total += (uint64_t)H.slice_w[sl] * 32;
    }
    H.col.assign(total, 0);
    H.val.assign(total * 4, 0);
    for (uint32_t sl = 0; sl < slices; ++sl) {
        for (uint32_t ln = 0; ln < 32; ++ln) {
            const uint64_t i = (uint64_t)sl * 32 + ln;
            if (i >= rows) break;
            const uint32_t r = order[i];
            H.perm[i] = r;
            for (uint32_t t = 0; t < len[r]; ++t) {
                const uint64_t src = (uint64_t)M.row_ptr[r] + t, dst = H.slice_off[sl] + (uint64_t)t * 32 + ln;
                H.col[dst] = M.col[src];
                memcpy(&H.val[dst * 4], M.val + src * 4, 32);
            }
        }
    }
    (void)ctx;
    return BZK_OK;
}

size_t sell_bytes(const SellHost &H) {
    return align_up(H.perm.size() * 4) + align_up(H.slice_w.size() * 4) + align_up(H.slice_off.size() * 8) +
           align_up(H.col.size() * 4) + align_up(H.val.size() * 8);
}

cudaError_t sell_upload(const SellHost &H, const bzk_csr &M, char *&cur, SellDev &D, cudaStream_t s) {
    D.rows = M.rows; D.cols = M.cols; D.slices = (uint32_t)H.slice_w.size(); D.entries = H.col.size();
    auto put = [&](const void *src, size_t n, auto *&dst) -> cudaError_t {
        dst = reinterpret_cast<std::remove_reference_t<decltype(dst)>>(cur);
        cur += align_up(n);
        return n ? cudaMemcpyAsync((void *)dst, src, n, cudaMemcpyHostToDevice, s) : cudaSuccess;
    };
    cudaError_t e;
    if ((e = put(H.perm.data(), H.perm.size() * 4, D.perm)) != cudaSuccess) return e;
    if ((e = put(H.slice_w.data(), H.slice_w.size() * 4, D.slice_w)) != cudaSuccess) return e;
    if ((e = put(H.slice_off.data(), H.slice_off.size() * 8, D.slice_off)) != cudaSuccess) return e;
    if ((e = put(H.col.data(), H.col.size() * 4, D.col)) != cudaSuccess) return e;
    if ((e = put(H.val.data(), H.val.size() * 8, D.val)) != cudaSuccess) return e;
    return enc_launch_to_mont(D.val, D.entries, s);
}

bzk_status encoder_create_impl(bzk_ctx *ctx, const bzk_code *c, bzk_encoder **out) {
    if (!c || !out) return fail(ctx, BZK_EINVAL, "code/out is NULL");
    *out = nullptr;
    if (c->log_n > 26) return fail(ctx, BZK_EINVAL, "log_n must be <= 26");
    const uint64_t n = 1ull << c->log_n;
    if (c->levels > 0 && (!c->A || !c->B)) return fail(ctx, BZK_EINVAL, "A/B is NULL");
    if (!c->G0) return fail(ctx, BZK_EINVAL, "G0 is NULL");
    // shapes (reading R21): A_l is n_l/4 x n_l, B_l is n_l/2 x n_l/2, G0 is n_L x n_L
    for (uint32_t l = 0; l < c->levels; ++l) {
        const uint64_t nl = n >> (2 * l);
        if (nl < 8 || c->A[l].cols != nl || c->A[l].rows != nl / 4 || c->B[l].cols != nl / 2 || c->B[l].rows != nl / 2)
            return fail(ctx, BZK_EINVAL, "graph shapes do not match log_n / level " + std::to_string(l));
    }
    const uint64_t m = n >> (2 * c->levels);
    if (m == 0 || c->G0->rows != m || c->G0->cols != m) return fail(ctx, BZK_EINVAL, "G0 must be n_L x n_L");
    std::vector<SellHost> HA(c->levels), HB(c->levels);
    SellHost HG;
    std::string why;
    size_t bytes = 0;
    for (uint32_t l = 0; l < c->levels; ++l) {
        if (sell_build(ctx, c->A[l], HA[l], why) || sell_build(ctx, c->B[l], HB[l], why))
            return fail(ctx, BZK_EINVAL, "level " + std::to_string(l) + ": " + why);
        bytes += sell_bytes(HA[l]) + sell_bytes(HB[l]);
    }
    if (sell_build(ctx, *c->G0, HG, why)) return fail(ctx, BZK_EINVAL, "G0: " + why);
    bytes += sell_bytes(HG);
    bzk_encoder *E = new bzk_encoder();
    E->device = ctx->device; E->log_n = c->log_n; E->levels = c->levels; E->m = (uint32_t)m; E->bytes = bytes;
    cudaError_t e = cudaMalloc(&E->mem, std::max<size_t>(bytes, 256));
    if (e != cudaSuccess) { cudaGetLastError(); delete E; return fail(ctx, BZK_ENOMEM, "cudaMalloc encoder graphs"); }
    char *cur = (char *)E->mem;
    E->A.resize(c->levels); E->B.resize(c->levels);
    cudaStream_t s = ctx->copy_stream;
    for (uint32_t l = 0; l < c->levels && e == cudaSuccess; ++l) {
        e = sell_upload(HA[l], c->A[l], cur, E->A[l], s);
        if (e == cudaSuccess) e = sell_upload(HB[l], c->B[l], cur, E->B[l], s);
    }
    if (e == cudaSuccess) e = sell_upload(HG, *c->G0, cur, E->G0, s);
    if (e == cudaSuccess) e = cudaStreamSynchronize(s);   // host SELL arrays die with this scope
    if (e != cudaSuccess) { cudaFree(E->mem); delete E; return cuda_fail(ctx, e, "encoder upload"); }
    *out = E;
    return BZK_OK;
}

cudaError_t spmv(bzk_ctx *ctx, const SellDev &M, const fe *src, fe *dst, uint64_t stride, uint64_t nb, cudaStream_t s) {
    const uint32_t warps = BZK_ENC_TPB / 32;   // slices per CTA
    const uint64_t per_launch = 65535ull * BZK_ENC_K;   // gridDim.y limit
    for (uint64_t c0 = 0; c0 < nb; c0 += per_launch) {
        const uint64_t n = std::min<uint64_t>(per_launch, nb - c0);
        enc::SpmvParams p;
        p.perm = M.perm; p.slice_off = M.slice_off; p.slice_w = M.slice_w; p.col = M.col; p.val = M.val;
        p.slices = M.slices; p.src = src + c0 * stride; p.dst = dst + c0 * stride; p.stride = stride; p.batch = n;
        dim3 grid((M.slices + warps - 1) / warps,
                  (uint32_t)((n + BZK_ENC_K - 1) / BZK_ENC_K));
        ProfScope ps_(ctx, s, 8);
        ++ctx->launches;
        cudaError_t e = enc_launch_spmv(grid, BZK_ENC_TPB, s, p);
        if (e != cudaSuccess) return e;
    }
    return cudaSuccess;
}

// encode nb codewords in place: C[b][0..n) = message on entry, C[b][0..2n) = codeword on exit
bzk_status encode_wave(bzk_ctx *ctx, const bzk_encoder *E, fe *C, uint64_t nb, cudaStream_t s) {
    const uint64_t n = 1ull << E->log_n, stride = 2 * n;
    std::vector<uint64_t> o(E->levels + 1), nl(E->levels + 1);
    o[0] = 0; nl[0] = n;
    for (uint32_t l = 0; l < E->levels; ++l) { o[l + 1] = o[l] + nl[l]; nl[l + 1] = nl[l] / 4; }
    for (uint32_t l = 0; l < E->levels; ++l)             // forward chain: x_{l+1} = A_l x_l
        CK(spmv(ctx, E->A[l], C + o[l], C + o[l + 1], stride, nb, s));
    const uint32_t L = E->levels;
    CK(spmv(ctx, E->G0, C + o[L], C + o[L] + nl[L], stride, nb, s));   // base: x_L || G0 x_L
    for (int l = (int)L - 1; l >= 0; --l)                 // reverse chain: w_l = B_l c_{l+1}
        CK(spmv(ctx, E->B[l], C + o[l + 1], C + o[l] + nl[l] + nl[l] / 2, stride, nb, s));
    return BZK_OK;
}

bzk_status encode_impl(bzk_ctx *ctx, const bzk_encoder *E, uint64_t *codes, uint64_t batch, uint32_t codes_mem,
                       uint32_t flags, cudaStream_t s) {
    NvtxRange nv_("bzk_encode");
    if (!E || !codes) return fail(ctx, BZK_EINVAL, "encoder/codes is NULL");
    if (E->device != ctx->device) return fail(ctx, BZK_EINVAL, "encoder belongs to another device");
    if (batch == 0) return fail(ctx, BZK_EINVAL, "batch must be >= 1");
    if (codes_mem > 1) return fail(ctx, BZK_EINVAL, "bad codes_mem");
    const uint64_t n = 1ull << E->log_n;
    const size_t cw = (size_t)2 * n * 32;   // bytes per codeword
    if (codes_mem == BZK_MEM_DEVICE) {
        if ((uintptr_t)codes & 31u) return fail(ctx, BZK_EINVAL, "device codes must be 32-byte aligned");
        bzk_status st = call_begin(ctx, s);
        if (st) return st;
        st = encode_wave(ctx, E, (fe *)codes, batch, s);
        if (st) return st;
        st = call_end(ctx, s);
        if (st) return st;
        if (flags & BZK_F_SYNC) CK(cudaStreamSynchronize(s));
        return BZK_OK;
    }
    // host codewords: waves through the loader ring (H2D of the messages on copy_stream, D2H of the
    // codewords on d2h_stream, overlapping the next wave's encoding)
    size_t limit = ctx->workspace_limit;
    if (limit == 0) {
        size_t fr = 0, tot = 0;
        cudaMemGetInfo(&fr, &tot);
        fr += 2 * ctx->stage_size;
        limit = fr > (2ull << 30) ? fr - (2ull << 30) : fr / 2;
    }
    uint64_t bw = batch;
    if (batch >= 8 && batch * cw > (1ull << 30)) bw = (batch + 7) / 8;
    while (bw > 1 && 2 * bw * cw + 4096 > limit) bw = (bw + 1) / 2;
    if (2 * bw * cw + 4096 > limit) return fail(ctx, BZK_ENOMEM, "workspace_limit too small for one codeword");
    const uint64_t nw = (batch + bw - 1) / bw;
    bw = (batch + nw - 1) / nw;
    bzk_status st = ensure_stage(ctx, align_up(bw * cw));
    if (st) return st;
    st = call_begin(ctx, s);
    if (st) return st;
    for (uint64_t w = 0; w < nw; ++w) {
        const uint64_t b0 = w * bw, nb = std::min<uint64_t>(bw, batch - b0);
        const int slot = ctx->next_slot;
        ctx->next_slot ^= 1;
        if (ctx->slot_used[slot]) CK(cudaStreamWaitEvent(ctx->copy_stream, ctx->ev_consumed[slot], 0));
        char *dev = (char *)ctx->stage[slot];
        {
            ProfScope ps_(ctx, ctx->copy_stream, 5);
            // messages only (the first n elements of every codeword)
            CK(cudaMemcpy2DAsync(dev, cw, (const char *)codes + b0 * cw, cw, n * 32, nb, cudaMemcpyHostToDevice,
                                 ctx->copy_stream));
        }
        CK(cudaEventRecord(ctx->ev_copied[slot], ctx->copy_stream));
        CK(cudaStreamWaitEvent(s, ctx->ev_copied[slot], 0));
        st = encode_wave(ctx, E, (fe *)dev, nb, s);
        if (st) return st;
        CK(cudaEventRecord(ctx->ev_nodes_ready[slot], s));
        CK(cudaStreamWaitEvent(ctx->d2h_stream, ctx->ev_nodes_ready[slot], 0));
        {
            ProfScope ps_(ctx, ctx->d2h_stream, 7);
            CK(cudaMemcpyAsync((char *)codes + b0 * cw, dev, nb * cw, cudaMemcpyDeviceToHost, ctx->d2h_stream));
        }
        CK(cudaEventRecord(ctx->ev_consumed[slot], ctx->d2h_stream));
        ctx->slot_used[slot] = true;
    }
    CK(cudaStreamSynchronize(ctx->d2h_stream));
    st = call_end(ctx, s);
    if (st) return st;
    CK(cudaStreamSynchronize(s));
    return BZK_OK;
}

// ---------------------------------------------------------------- the section-4 chain (NEXT-4)
//
// P:207-213 (Fig. 7): each proof's input is divided into segments, each segment is encoded, every
// codeword is committed with a Merkle tree, the codeword roots are the leaves of another tree whose
// root seeds the sum-check's random numbers.  One call runs the chain over a batch of proofs, every
// step in the library's kernels, stream-ordered (no host round trip between the modules).

bzk_status commit_prove_impl(bzk_ctx *ctx, const bzk_encoder *E, const bzk_commit *c, const bzk_batch *sc,
                             cudaStream_t s) {
    NvtxRange nv_("bzk_commit_prove");
    if (!E || !c || !sc) return fail(ctx, BZK_EINVAL, "encoder/commit/sumcheck is NULL");
    if (!c->codes || !c->roots || !c->final_roots) return fail(ctx, BZK_EINVAL, "codes/roots/final_roots is NULL");
    const uint32_t S = c->segments;
    if (S == 0 || (S & (S - 1)) || S > (1u << 20)) return fail(ctx, BZK_EINVAL, "segments must be a power of two <= 2^20");
    if (c->hash > 1) return fail(ctx, BZK_EINVAL, "hash must be BZK_MERKLE_COMPRESS or BZK_MERKLE_SHA256");
    if (sc->flags & (BZK_F_SEEDS_DEVICE | BZK_F_GIVEN_CHALLENGES | BZK_F_FIELD_GOLDILOCKS))
        return fail(ctx, BZK_EINVAL, "the chain derives the seeds: no SEEDS_DEVICE / GIVEN_CHALLENGES / GOLDILOCKS");
    if (sc->tables_mem != BZK_MEM_DEVICE || sc->outputs_mem != BZK_MEM_DEVICE)
        return fail(ctx, BZK_EINVAL, "bzk_commit_prove takes device buffers");
    auto mis = [](const void *q) { return q && ((uintptr_t)q & 31u); };
    if (mis(c->codes) || mis(c->roots) || mis(c->nodes) || mis(c->final_roots))
        return fail(ctx, BZK_EINVAL, "device buffers must be 32-byte aligned");
    if (E->device != ctx->device) return fail(ctx, BZK_EINVAL, "encoder belongs to another device");
    bzk_batch b2 = *sc;                  // the sum-check, its transcripts seeded with the final roots
    b2.flags |= BZK_F_SEEDS_DEVICE;
    b2.seed = c->final_roots;
    bzk_status st = validate_args(ctx, &b2);   // every argument error before the first launch
    if (st) return st;
    const uint64_t B = sc->batch, n = 1ull << E->log_n;
    const uint32_t lg = [&] { uint32_t l = 0; while ((2u << l) < S) ++l; return l; }();   // top tree: S/2 blocks
    // Module pipeline over proof chunks (P:207-213 run as stages, "all pipelined modules are fully
    // engaged ... concurrently"): chunk j is encoded on the caller's stream while chunk j-1 is committed
    // on a Merkle stream (ALU-pipe work beside the encoder's IMAD work) and chunk j-2 is proved on a
    // sum-check stream; events order each chunk's three steps.
    const uint64_t Bc = (B + std::min<uint64_t>(B, knobs().chain_chunks) - 1) / std::min<uint64_t>(B, knobs().chain_chunks);
    const uint64_t nc = (B + Bc - 1) / Bc;   // chunks actually used (B = 5 in chunks of 2: 3 chunks)
    const std::vector<MkStage> st1 = merkle_stages(E->log_n);
    const std::vector<MkStage> st2 = merkle_stages(lg);
    const size_t spt1 = c->nodes ? 0 : (size_t)32 << st1[0].lg_tpt, spt2 = (size_t)32 << st2[0].lg_tpt;
    const size_t scr1 = align_up(Bc * S * spt1), scr2 = align_up(Bc * spt2);
    const size_t chain_bytes = 2 * scr1 + 2 * scr2 + 256;
    std::vector<Plan> plans(nc);
    size_t ws_need = 0;
    for (uint64_t j = 0; j < nc; ++j) {
        bzk_batch bj = b2;
        bj.batch = std::min<uint64_t>(Bc, B - j * Bc);
        st = make_plan(ctx, &bj, plans[j]);
        if (st) return st;
        ws_need = std::max(ws_need, plans[j].total);
    }
    st = ensure_ws(ctx, ws_need);
    if (st) return st;
    if (ctx->chain_ws_size < chain_bytes) {
        cudaDeviceSynchronize();
        if (ctx->chain_ws) cudaFree(ctx->chain_ws);
        ctx->chain_ws = nullptr;
        ctx->chain_ws_size = 0;
        if (cudaMalloc(&ctx->chain_ws, chain_bytes) != cudaSuccess) {
            cudaGetLastError();
            return fail(ctx, BZK_ENOMEM, "cudaMalloc chain scratch");
        }
        ctx->chain_ws_size = chain_bytes;
    }
    if (!ctx->chain_mk) CK(cudaStreamCreateWithFlags(&ctx->chain_mk, cudaStreamNonBlocking));
    if (!ctx->chain_sc) CK(cudaStreamCreateWithFlags(&ctx->chain_sc, cudaStreamNonBlocking));
    cudaStream_t smk = ctx->chain_mk, ssc = ctx->chain_sc;
    st = call_begin(ctx, s);
    if (st) return st;
    std::vector<cudaEvent_t> evs;
    auto ev = [&]() { cudaEvent_t e = pool_event(ctx); evs.push_back(e); return e; };
    auto join = [&](cudaStream_t from, cudaStream_t to) -> bzk_status {
        cudaEvent_t e = ev();
        CK(cudaEventRecord(e, from));
        CK(cudaStreamWaitEvent(to, e, 0));
        return BZK_OK;
    };
    if ((st = join(s, smk)) || (st = join(s, ssc))) return st;
    char *cw = (char *)ctx->chain_ws;
    uint8_t *const scrA[2] = {(uint8_t *)cw, (uint8_t *)cw + scr1};
    uint8_t *const scrB[2] = {(uint8_t *)cw + 2 * scr1, (uint8_t *)cw + 2 * scr1 + scr2};
    const size_t cw_elems = 2 * n, nodes_bytes = (size_t)(2 * n - 1) * 32;
    const size_t tbl_words = (size_t)sc->degree * ((size_t)1 << sc->num_vars) * 4;
    for (uint64_t j = 0; j < nc; ++j) {
        const uint64_t b0 = j * Bc, bc = std::min<uint64_t>(Bc, B - b0);
        fe *codes_j = (fe *)c->codes + b0 * S * cw_elems;
        uint8_t *roots_j = c->roots + b0 * S * 32, *fin_j = c->final_roots + b0 * 32;
        // 1. encode (caller's stream)
        st = encode_wave(ctx, E, codes_j, bc * S, s);
        if (st) return st;
        if ((st = join(s, smk))) return st;
        // 2. codeword trees + root of roots (Merkle stream)
        st = merkle_chain(ctx, c->hash, E->log_n, st1, (const uint8_t *)codes_j, cw_elems * 32,
                          c->nodes ? c->nodes + b0 * S * nodes_bytes : nullptr, nodes_bytes, roots_j, scrA, spt1,
                          bc * S, smk);
        if (st) return st;
        if (S == 1) CK(cudaMemcpyAsync(fin_j, roots_j, bc * 32, cudaMemcpyDeviceToDevice, smk));
        else {
            st = merkle_chain(ctx, c->hash, lg, st2, roots_j, (uint64_t)S * 32, nullptr, 0, fin_j, scrB, spt2, bc, smk);
            if (st) return st;
        }
        if ((st = join(smk, ssc))) return st;
        // 3. the chunk's sum-checks, seeded with their final roots (sum-check stream)
        bzk_batch bj = b2;
        bj.batch = bc;
        bj.first_index = b2.first_index + b0;
        bj.seed = fin_j;
        bj.tables = b2.tables + b0 * tbl_words;
        bj.round_evals = b2.round_evals + b0 * (size_t)sc->num_vars * (sc->degree + 1) * 4;
        bj.challenges = b2.challenges + b0 * (size_t)sc->num_vars * 4;
        bj.final_evals = b2.final_evals + b0 * (size_t)sc->degree * 4;
        bj.claims = b2.claims ? b2.claims + b0 * 4 : nullptr;
        st = enqueue_job(ctx, &bj, plans[j], ssc);
        if (st) return st;
    }
    if ((st = join(smk, s)) || (st = join(ssc, s))) return st;
    for (auto e : evs) ctx->ev_pool.push_back(e);
    st = call_end(ctx, s);
    if (st) return st;
    if (sc->flags & BZK_F_SYNC) CK(cudaStreamSynchronize(s));
    return BZK_OK;
}

// ---------------------------------------------------------------- debug kernels

__global__ void k_debug_field(int op, uint64_t n, const fe *a, const fe *b, fe *out) {
    for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n;
         i += (uint64_t)gridDim.x * blockDim.x) {
        fe x = ld_fe(a + i), r;
        switch (op) {
            case 0: r = fe_add(x, ld_fe(b + i)); break;
            case 1: r = fe_sub(x, ld_fe(b + i)); break;
            case 2: r = mont_mul(x, ld_fe(b + i)); break;
            case 3: r = mont_mul(mont_mul(x, ld_fe(b + i)), fe_const(2)); break;
            case 5: { f6 fx = to_f6(x), fy = to_f6(ld_fe(b + i)); r = fmont<1>(fx, fy, fx, fy); break; }
            case 6: { f6 fx = to_f6(x), fy = to_f6(ld_fe(b + i)); r = fmont<2>(fx, fy, fy, fx); break; }
            default: r = fe_reduce_256(x); break;
        }
        st_fe(out + i, r);
    }
}

// Lazy hot-path primitives at their stated operand bounds (bzk_debug_field ops 7..16; the results are
// the RAW lazy values, so the host can check both the congruence and the bound).  64 threads per CTA:
// fixmul_lz reads its table K from shared memory.
__global__ void __launch_bounds__(64) k_debug_lazy(int op, uint64_t n, const fe *a, const fe *b, fe *out, uint32_t zero) {
    __shared__ __align__(16) fe sK[64][8];
    for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x) {
        const fe x = ld_fe(a + i), y = ld_fe(b + i);
        fe r;
        switch (op) {
            case 7: r = mont_mul_lz(x, y); break;                                       // x y R^-1 + q p
            case 8: r = mont_mul2_lz(x, y, ld_fe(a + n - 1 - i), ld_fe(b + n - 1 - i)); break;
            case 9: case 16: {                                                          // K_j = r 2^(32 j + 64)
                const fe rr = op == 9 ? y : ld_fe(b + n + i);
                const fe rm = mont_mul(rr, fe_const(2));                                // r R
                fe pw = fe_zero();
                pw.l[0] = 1;
                for (int e = 0; e < 64; ++e) pw = fe_add(pw, pw);                      // 2^64 mod p
                for (int j = 0; j < 8; ++j) {
                    sK[threadIdx.x][j] = mont_mul(rm, pw);
                    for (int e = 0; e < 32; ++e) pw = fe_add(pw, pw);
                }
                __syncwarp();
                r = op == 9 ? fixmul_lz(x, sK[threadIdx.x], zero) : fold_fx(x, y, sK[threadIdx.x], zero);
                __syncwarp();
                break;
            }
            case 10: {                                                                  // sum of 64 products
                acc17 acc = acc17_zero();
                for (uint64_t j = 0; j < 64; ++j) mul_acc(acc, ld_fe(a + (i + j) % n), ld_fe(b + (i + j) % n));
                r = acc17_to_fe(acc);
                break;
            }
            case 11: {                                                                  // raw 544-bit value
                acc17 acc;
                for (int w = 0; w < 8; ++w) { acc.w[w] = x.l[w]; acc.w[8 + w] = y.l[w]; }
                acc.w[16] = x.l[7];
                r = acc17_to_fe(acc);
                break;
            }
            case 12: r = lz_sub(y, x); break;                                           // y + 2p - x
            case 13: r = lz_red(x); break;                                              // x < 4p -> < 2p
            case 14: { acc9 c; c.lo = x; c.hi = y.l[0]; r = acc9_to_fe(c); break; }   // lo + hi 2^256
            default: r = lz_add(x, y); break;                                           // 15: plain add
        }
        st_fe(out + i, r);
    }
}

// Goldilocks primitives (gl.cuh), bzk_debug_gl
__global__ void k_debug_gl(int op, uint64_t n, const uint64_t *a, const uint64_t *b, uint64_t *out) {
    for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x) {
        const uint64_t x = a[i], y = b[i];
        uint64_t r;
        switch (op) {
            case 0: r = gl::add(x, y); break;
            case 1: r = gl::sub(x, y); break;
            case 2: r = gl::mul(x, y); break;
            case 3: r = gl::add_lazy(x, y); break;
            case 4: r = gl::reduce128(x, y); break;                                   // x = hi, y = lo
            case 5: r = gl::fold(x, y, b[n + i]); break;                                // x + r (y - x)
            case 6: {                                                                   // 64 products, lazy
                gl::Wide w{0, 0, 0};
                for (uint64_t j = 0; j < 64; ++j) gl::wide_mac(w, a[(i + j) % n], b[(i + j) % n]);
                r = gl::wide_reduce(w);
                break;
            }
            default: r = gl::wide_reduce(gl::Wide{x, y, b[n + i] & 0xffffffffull}); break;   // 7: raw 160-bit
        }
        out[i] = r;
    }
}

__global__ void k_debug_sha256(const uint8_t *msgs, uint32_t len, uint64_t n, uint8_t *out) {
    uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= n) return;
    const uint8_t *m = msgs + i * len;
    sha256_words sh;
    sh.init();
    for (uint32_t w = 0; w < len / 4; ++w)
        sh.push(((uint32_t)m[4 * w] << 24) | ((uint32_t)m[4 * w + 1] << 16) | ((uint32_t)m[4 * w + 2] << 8) |
                (uint32_t)m[4 * w + 3]);
    uint32_t h[8];
    sh.finish(h);
    for (int j = 0; j < 8; ++j) {
        out[i * 32 + 4 * j] = (uint8_t)(h[j] >> 24);
        out[i * 32 + 4 * j + 1] = (uint8_t)(h[j] >> 16);
        out[i * 32 + 4 * j + 2] = (uint8_t)(h[j] >> 8);
        out[i * 32 + 4 * j + 3] = (uint8_t)h[j];
    }
}

// Micro-benchmarks that calibrate the integer roof (bzk_debug_bench).
//   kind 0: mad.lo.u32 (IMAD)      kind 1: mul.wide.u32 (IMAD.WIDE.U32)
//   kind 2: mont_mul_v1            kind 3: mont_mul (hot path)
template <int KIND>
__global__ void __launch_bounds__(256, 2) k_bench(uint32_t iters, uint32_t seed, uint32_t *sink) {
    const uint32_t tid = blockIdx.x * blockDim.x + threadIdx.x;
    if (KIND == 4) {   // DFMA throughput (FP64 pipe)
        double a[8];
#pragma unroll
        for (int i = 0; i < 8; ++i) a[i] = 1.0 + 1e-9 * (tid + i);
        const double x = 0.999999, y = 1e-7 * (seed & 7);
        for (uint32_t it = 0; it < iters; ++it) {
#pragma unroll
            for (int u = 0; u < 4; ++u)
#pragma unroll
                for (int i = 0; i < 8; ++i) asm volatile("fma.rn.f64 %0, %0, %1, %2;" : "+d"(a[i]) : "d"(x), "d"(y));
        }
        double acc = 0;
#pragma unroll
        for (int i = 0; i < 8; ++i) acc += a[i];
        sink[tid] = (uint32_t)__double2loint(acc);
        return;
    }
    if (KIND <= 1) {
        uint32_t a[8];
        uint64_t w[8];
#pragma unroll
        for (int i = 0; i < 8; ++i) { a[i] = seed ^ (tid + i); w[i] = a[i]; }
        const uint32_t x = seed | 1, y = seed >> 3;
        for (uint32_t it = 0; it < iters; ++it) {
#pragma unroll
            for (int u = 0; u < 4; ++u)
#pragma unroll
                for (int i = 0; i < 8; ++i) {
                    if (KIND == 0) asm volatile("mad.lo.u32 %0, %0, %1, %2;" : "+r"(a[i]) : "r"(x), "r"(y));
                    else asm volatile("mad.wide.u32 %0, %1, %2, %0;" : "+l"(w[i]) : "r"((uint32_t)w[i]), "r"(x));
                }
        }
        uint32_t acc = 0;
#pragma unroll
        for (int i = 0; i < 8; ++i) acc ^= a[i] ^ (uint32_t)w[i] ^ (uint32_t)(w[i] >> 32);
        sink[tid] = acc;
    } else {
        constexpr int CH = KIND == 5 ? 1 : (KIND == 6 ? 2 : (KIND >= 9 ? 2 : 4));
        fe x[4], y;
#pragma unroll
        for (int c = 0; c < 4; ++c)
#pragma unroll
            for (int i = 0; i < 8; ++i) x[c].l[i] = (seed * (i + 1) + tid * 7 + c) & (i == 7 ? 0x0fffffffu : ~0u);
#pragma unroll
        for (int i = 0; i < 8; ++i) y.l[i] = (seed ^ (0x9e3779b9u * (i + 3))) & (i == 7 ? 0x0fffffffu : ~0u);
        for (uint32_t it = 0; it < iters; ++it)
#pragma unroll
            for (int c = 0; c < CH; ++c) {
                // 9: FP64 only; 10: odd warps FP64, even warps IMAD; 11: each thread alternates
                const bool fp = KIND == 9 || (KIND == 10 && ((threadIdx.x >> 5) & 1)) || (KIND == 11 && (c & 1));
                if (KIND >= 9 && fp) {
                    const f6 a = to_f6(x[c]), b = to_f6(y), u = to_f6(x[(c + 1) & 3]);
                    x[c] = fmont<2>(a, b, u, b);
                } else if (KIND >= 9) x[c] = mont_mul2(x[c], y, x[(c + 1) & 3], y);
                else if (KIND == 2) x[c] = mont_mul_v1(x[c], y);
                else if (KIND == 8) x[c] = mont_mul2(x[c], y, x[(c + 1) & 3], y);
                else x[c] = mont_mul(x[c], y);
            }
        uint32_t acc = 0;
#pragma unroll
        for (int c = 0; c < 4; ++c)
#pragma unroll
            for (int i = 0; i < 8; ++i) acc ^= x[c].l[i];
        sink[tid] = acc;
    }
}

}  // namespace

// ==== (see below)
namespace {
template <int KIND>
cudaError_t run_bench(uint32_t iters, double *rate, cudaStream_t s) {
    int nsm = kSMs, clk_khz = 1965000;
    cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0);
    cudaDeviceGetAttribute(&clk_khz, cudaDevAttrClockRate, 0);
    // kinds 5-7: 2 CTAs of 256 threads per SM (the occupancy of k_round) with 1 / 2 / 4 chains per thread
    const int threads = 256, blocks = (KIND >= 5 && KIND <= 7) ? nsm * 2 : nsm * 8;
    uint32_t *sink = nullptr;
    cudaError_t e = cudaMalloc(&sink, (size_t)blocks * threads * 4);
    if (e != cudaSuccess) return e;
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    k_bench<KIND><<<blocks, threads, 0, s>>>(iters / 8 + 1, 12345u, sink);   // warm-up
    cudaEventRecord(e0, s);
    k_bench<KIND><<<blocks, threads, 0, s>>>(iters, 12345u, sink);
    cudaEventRecord(e1, s);
    e = cudaEventSynchronize(e1);
    float ms = 0;
    cudaEventElapsedTime(&ms, e0, e1);
    cudaEventDestroy(e0);
    cudaEventDestroy(e1);
    cudaFree(sink);
    const double per = (KIND <= 1 || KIND == 4) ? 32.0 : (KIND == 5 ? 1.0 : ((KIND == 6 || KIND >= 9) ? 2.0 : 4.0));
    const double ops = (double)blocks * threads * iters * per;   // kind 8 counts mont_mul2 calls
    *rate = ops / (ms * 1e-3) / ((double)clk_khz * 1e3) / nsm;   // per SM per clock (at the max clock)
    return e;
}
}  // namespace

// ==================================================================== C ABI

extern "C" {

const char *bzk_version(void) { return "bzk 0.4 sm_100a (BN254 Fr + Goldilocks sum-check, SHA-256 Fiat-Shamir, TMA-staged rounds, cluster small-batch kernel, known-challenge multi-round passes, batched Merkle trees, linear-time encoder, section-4 chain)"; }

const char *bzk_strerror(bzk_status s) {
    switch (s) {
        case BZK_OK: return "ok";
        case BZK_EINVAL: return "invalid argument";
        case BZK_ENOMEM: return "out of device memory / workspace limit";
        case BZK_ECUDA: return "CUDA error";
        case BZK_ENONCANON: return "non-canonical input element";
        case BZK_EUNSUPPORTED: return "unsupported";
    }
    return "unknown status";
}

const char *bzk_last_error(const bzk_ctx *ctx) { return ctx ? ctx->last_error.c_str() : ""; }

}  // extern "C"

namespace {
// frees everything a (possibly partially constructed) context owns
void ctx_free(bzk_ctx *ctx) {
    if (ctx->ws) cudaFree(ctx->ws);
    if (ctx->d_flag) cudaFree(ctx->d_flag);
    if (ctx->consts) cudaFree(ctx->consts);
    for (int i = 0; i < 2; ++i)
        if (ctx->stage[i]) cudaFree(ctx->stage[i]);
    for (int i = 0; i < 2; ++i) {
        if (ctx->ev_copied[i]) cudaEventDestroy(ctx->ev_copied[i]);
        if (ctx->ev_consumed[i]) cudaEventDestroy(ctx->ev_consumed[i]);
        if (ctx->ev_nodes_ready[i]) cudaEventDestroy(ctx->ev_nodes_ready[i]);
        if (ctx->ev_nodes_copied[i]) cudaEventDestroy(ctx->ev_nodes_copied[i]);
    }
    if (ctx->ev_done) cudaEventDestroy(ctx->ev_done);
    if (ctx->chain_mk) cudaStreamDestroy(ctx->chain_mk);
    if (ctx->dual_stream) cudaStreamDestroy(ctx->dual_stream);
    if (ctx->chain_sc) cudaStreamDestroy(ctx->chain_sc);
    if (ctx->chain_ws) cudaFree(ctx->chain_ws);
    if (ctx->d2h_stream) cudaStreamDestroy(ctx->d2h_stream);
    if (ctx->graph_exec) cudaGraphExecDestroy(ctx->graph_exec);
    for (auto &r : ctx->recs) { cudaEventDestroy(r.a); cudaEventDestroy(r.b); }
    for (auto e : ctx->ev_pool) cudaEventDestroy(e);
    if (ctx->copy_stream) cudaStreamDestroy(ctx->copy_stream);
    delete ctx;
}
}  // namespace

extern "C" {

bzk_status bzk_create(int device, size_t workspace_limit, bzk_ctx **out) {
    if (!out) return BZK_EINVAL;
    *out = nullptr;
    int n = 0;
    cudaError_t e = cudaGetDeviceCount(&n);
    if (e != cudaSuccess || n == 0) return BZK_ECUDA;
    if (device < 0 || device >= n) return BZK_EINVAL;
    e = cudaSetDevice(device);
    if (e != cudaSuccess) return BZK_ECUDA;
    bzk_ctx *ctx = new bzk_ctx();
    ctx->device = device;
    ctx->workspace_limit = workspace_limit;
    cudaDeviceGetAttribute(&ctx->num_sms, cudaDevAttrMultiProcessorCount, device);
    bool ok = cudaStreamCreateWithFlags(&ctx->copy_stream, cudaStreamNonBlocking) == cudaSuccess &&
              cudaStreamCreateWithFlags(&ctx->d2h_stream, cudaStreamNonBlocking) == cudaSuccess &&
              cudaMalloc(&ctx->d_flag, 4) == cudaSuccess &&
              cudaMalloc(&ctx->consts, sizeof(fe) * kNumConsts) == cudaSuccess &&
              cudaEventCreateWithFlags(&ctx->ev_done, cudaEventDisableTiming) == cudaSuccess;
    for (int i = 0; ok && i < 2; ++i)
        ok = cudaEventCreateWithFlags(&ctx->ev_copied[i], cudaEventDisableTiming) == cudaSuccess &&
             cudaEventCreateWithFlags(&ctx->ev_consumed[i], cudaEventDisableTiming) == cudaSuccess &&
             cudaEventCreateWithFlags(&ctx->ev_nodes_ready[i], cudaEventDisableTiming) == cudaSuccess &&
             cudaEventCreateWithFlags(&ctx->ev_nodes_copied[i], cudaEventDisableTiming) == cudaSuccess;
    if (ok) {
        set_kernel_attrs<1>();
        set_kernel_attrs<2>();
        set_kernel_attrs<3>();
        set_kernel_attrs<4>();
        gl_set_attrs();
        multi_set_attrs();
        r1tc_set_attrs();
        k_init_consts<<<1, 32, 0, ctx->copy_stream>>>(ctx->consts);
        ok = cudaStreamSynchronize(ctx->copy_stream) == cudaSuccess;
    }
    if (!ok) {
        cudaGetLastError();
        ctx_free(ctx);
        return BZK_ECUDA;
    }
    *out = ctx;
    return BZK_OK;
}

void bzk_destroy(bzk_ctx *ctx) {
    if (!ctx) return;
    cudaSetDevice(ctx->device);
    cudaDeviceSynchronize();
    ctx_free(ctx);
}

bzk_status bzk_workspace_size(bzk_ctx *ctx, const bzk_batch *batch, size_t *bytes) {
    if (!ctx || !bytes) return BZK_EINVAL;
    bzk_status st = validate_args(ctx, batch);
    if (st) return st;
    Plan P;
    st = make_plan(ctx, batch, P);
    if (st) return st;
    *bytes = P.total + 2 * P.stage_bytes;   // workspace + the loader's two staging slots (host tables)
    return BZK_OK;
}

bzk_status bzk_prove(bzk_ctx *ctx, const bzk_batch *batch, void *cuda_stream) {
    if (!ctx) return BZK_EINVAL;
    cudaSetDevice(ctx->device);
    if (!batch) return fail(ctx, BZK_EINVAL, "batch is NULL");
    return prove_jobs(ctx, batch, 1, (cudaStream_t)cuda_stream);
}

bzk_status bzk_prove_ragged(bzk_ctx *ctx, const bzk_batch *jobs, size_t njobs, void *cuda_stream) {
    if (!ctx || (!jobs && njobs)) return BZK_EINVAL;
    cudaSetDevice(ctx->device);
    return prove_jobs(ctx, jobs, njobs, (cudaStream_t)cuda_stream);
}

bzk_status bzk_sync(bzk_ctx *ctx) {
    if (!ctx) return BZK_EINVAL;
    cudaSetDevice(ctx->device);
    cudaError_t e = cudaDeviceSynchronize();
    if (e != cudaSuccess) return cuda_fail(ctx, e, "bzk_sync");
    e = cudaGetLastError();
    if (e != cudaSuccess) return cuda_fail(ctx, e, "bzk_sync");
    return BZK_OK;
}

bzk_status bzk_generate(uint64_t *dst, uint64_t batch, uint32_t d, uint32_t k, uint64_t first_index,
                        uint32_t dist, uint64_t data_seed, void *cuda_stream) {
    if (!dst || k > 30 || d < 1 || d > 15 || dist > 5 || first_index + batch > (1ull << 28)) return BZK_EINVAL;
    k_generate<<<kSMs * 16, 256, 0, (cudaStream_t)cuda_stream>>>(dst, batch, d, k, first_index, dist, data_seed);
    return cudaGetLastError() == cudaSuccess ? BZK_OK : BZK_ECUDA;
}

bzk_status bzk_merkle(bzk_ctx *ctx, const bzk_merkle_batch *batch, void *cuda_stream) {
    if (!ctx) return BZK_EINVAL;
    cudaSetDevice(ctx->device);
    return merkle_impl(ctx, batch, (cudaStream_t)cuda_stream);
}

bzk_status bzk_encoder_create(bzk_ctx *ctx, const bzk_code *code, bzk_encoder **out) {
    if (!ctx) return BZK_EINVAL;
    cudaSetDevice(ctx->device);
    return encoder_create_impl(ctx, code, out);
}

void bzk_encoder_destroy(bzk_encoder *enc) {
    if (!enc) return;
    cudaSetDevice(enc->device);
    cudaDeviceSynchronize();
    if (enc->mem) cudaFree(enc->mem);
    delete enc;
}

bzk_status bzk_encode(bzk_ctx *ctx, const bzk_encoder *enc, uint64_t *codes, uint64_t batch, uint32_t codes_mem,
                      uint32_t flags, void *cuda_stream) {
    if (!ctx) return BZK_EINVAL;
    cudaSetDevice(ctx->device);
    return encode_impl(ctx, enc, codes, batch, codes_mem, flags, (cudaStream_t)cuda_stream);
}

bzk_status bzk_commit_prove(bzk_ctx *ctx, const bzk_encoder *enc, const bzk_commit *commit, const bzk_batch *sumcheck,
                            void *cuda_stream) {
    if (!ctx) return BZK_EINVAL;
    cudaSetDevice(ctx->device);
    return commit_prove_impl(ctx, enc, commit, sumcheck, (cudaStream_t)cuda_stream);
}

bzk_status bzk_generate_blocks(uint8_t *dst, uint64_t batch, uint32_t n, uint64_t first_index, uint64_t data_seed,
                               void *cuda_stream) {
    if (!dst || n > 30 || batch == 0 || first_index + batch > (1ull << 28) || ((uintptr_t)dst & 7u)) return BZK_EINVAL;
    k_generate_blocks<<<kSMs * 16, 256, 0, (cudaStream_t)cuda_stream>>>((uint64_t *)dst, batch, n, first_index,
                                                                       data_seed);
    return cudaGetLastError() == cudaSuccess ? BZK_OK : BZK_ECUDA;
}

bzk_status bzk_profile_enable(bzk_ctx *ctx, int on) {
    if (!ctx) return BZK_EINVAL;
    ctx->prof = on != 0;
    return BZK_OK;
}

bzk_status bzk_profile_read(bzk_ctx *ctx, double ms[BZK_PROF_KINDS], uint64_t count[BZK_PROF_KINDS], int reset) {
    if (!ctx || !ms || !count) return BZK_EINVAL;
    cudaSetDevice(ctx->device);
    cudaError_t e = cudaDeviceSynchronize();
    if (e != cudaSuccess) return cuda_fail(ctx, e, "bzk_profile_read");
    for (int i = 0; i < BZK_PROF_KINDS; ++i) { ms[i] = 0; count[i] = 0; }
    for (auto &r : ctx->recs) {
        float t = 0;
        cudaEventElapsedTime(&t, r.a, r.b);
        if (r.kind >= 0 && r.kind < BZK_PROF_KINDS) { ms[r.kind] += t; count[r.kind] += 1; }
    }
    if (reset) {
        for (auto &r : ctx->recs) { ctx->ev_pool.push_back(r.a); ctx->ev_pool.push_back(r.b); }
        ctx->recs.clear();
    }
    return BZK_OK;
}

uint64_t bzk_launch_count(bzk_ctx *ctx, int reset) {
    if (!ctx) return 0;
    uint64_t n = ctx->launches;
    if (reset) ctx->launches = 0;
    return n;
}

bzk_status bzk_debug_field(int op, uint64_t n, const uint64_t *a, const uint64_t *b, uint64_t *out,
                           void *cuda_stream) {
    if (op < 0 || op > 16 || !a || !out || (op != 4 && !b)) return BZK_EINVAL;
    if (n == 0) return BZK_OK;
    if (op >= 7) {
        k_debug_lazy<<<kSMs * 4, 64, 0, (cudaStream_t)cuda_stream>>>(op, n, (const fe *)a, (const fe *)b, (fe *)out, 0u);
        return cudaGetLastError() == cudaSuccess ? BZK_OK : BZK_ECUDA;
    }
    k_debug_field<<<kSMs * 8, 256, 0, (cudaStream_t)cuda_stream>>>(op, n, (const fe *)a, (const fe *)b, (fe *)out);
    return cudaGetLastError() == cudaSuccess ? BZK_OK : BZK_ECUDA;
}

bzk_status bzk_debug_gl(int op, uint64_t n, const uint64_t *a, const uint64_t *b, uint64_t *out, void *cuda_stream) {
    if (op < 0 || op > 7 || !a || !b || !out) return BZK_EINVAL;
    if (n == 0) return BZK_OK;
    k_debug_gl<<<kSMs * 8, 256, 0, (cudaStream_t)cuda_stream>>>(op, n, a, b, out);
    return cudaGetLastError() == cudaSuccess ? BZK_OK : BZK_ECUDA;
}

bzk_status bzk_debug_sha256(const uint8_t *msgs, uint32_t msg_len, uint64_t n, uint8_t *out, void *cuda_stream) {
    if (!msgs || !out || msg_len % 4) return BZK_EINVAL;
    if (n == 0) return BZK_OK;
    k_debug_sha256<<<(uint32_t)((n + 127) / 128), 128, 0, (cudaStream_t)cuda_stream>>>(msgs, msg_len, n, out);
    return cudaGetLastError() == cudaSuccess ? BZK_OK : BZK_ECUDA;
}

bzk_status bzk_debug_bench(int kind, uint32_t iters, double *rate, void *cuda_stream) {
    if (!rate || iters == 0 || kind < 0 || kind > 11) return BZK_EINVAL;
    cudaStream_t s = (cudaStream_t)cuda_stream;
    cudaError_t e = cudaErrorInvalidValue;
    switch (kind) {
        case 0: e = run_bench<0>(iters, rate, s); break;
        case 1: e = run_bench<1>(iters, rate, s); break;
        case 2: e = run_bench<2>(iters, rate, s); break;
        case 3: e = run_bench<3>(iters, rate, s); break;
        case 4: e = run_bench<4>(iters, rate, s); break;
        case 5: e = run_bench<5>(iters, rate, s); break;
        case 6: e = run_bench<6>(iters, rate, s); break;
        case 7: e = run_bench<7>(iters, rate, s); break;
        case 8: e = run_bench<8>(iters, rate, s); break;
        case 9: e = run_bench<9>(iters, rate, s); break;
        case 10: e = run_bench<10>(iters, rate, s); break;
        case 11: e = run_bench<11>(iters, rate, s); break;
    }
    return e == cudaSuccess ? BZK_OK : BZK_ECUDA;
}

}  // extern "C"
