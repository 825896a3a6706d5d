// engine_batch.cu — SURVEY §8(f) NEXT-2: batched multi-source relaxation.  Q independent
// queries of one kind (vertex queries are independent) run through Alg 3
// in lock-step on one persistent kernel:
//
//   * values live as a ROW per vertex holding all Q queries' values, so ONE gather of v's row
//     serves the Needed test of every query: the random-access cost that bounds the
//     single-query sweep (one 32 B sector per edge per query) is shared by the batch;
//   * rows are packed by value lanes (Lanes32 / Lanes16 / LanesBit below): u32 lanes (the
//     Table 6 types; Viterbi, and the fallback of every kind) with Q = 16 — a 64 B row; binary16
//     lanes (SSSP / SSWP / SSNP / BFS: small integers, exact) with Q = 32 — a 64 B row; one bit
//     per query (REACH) with Q = 32 — a 4 B row.  The EdgeFunction of 8 binary16 lanes is one
//     vector red.min/max (REDG.F16x8), of 32 bit lanes one red.or;
//   * the frontier is the union over the batch: a vertex bitmap plus a per-vertex mask M[v]
//     of the queries for which v is active; phase 1 / phase 2 switch when the union converges;
//   * S1 / S2 as in engine.cu: CTA-aggregated compaction into an edge-offset list, the
//     iteration's edges split evenly over all warps; a lane takes one edge for all Q queries,
//     its value row copied global -> shared (cp.async) one 32-edge chunk ahead;
//   * finally the batch is transposed into the caller's [query][vertex] u32 layout.
#include <cstdio>
#include <cstdlib>

#include <cuda_fp16.h>
#include <type_traits>

#include "kernels.cuh"

namespace cgb {

namespace {

using namespace kern;

#ifndef CGB_BT
#define CGB_BT 512
#endif
constexpr int BT = CGB_BT;       // threads per CTA
constexpr int BW = BT / 32;      // warps per CTA
#ifndef CGB_STAGES
#define CGB_STAGES 2
#endif
constexpr int S_PIPE = CGB_STAGES;  // value-row pipeline depth (chunks of 32 edges per warp)
#ifndef CGB_EAHEAD
#define CGB_EAHEAD CGB_STAGES
#endif
constexpr int E_AHEAD = CGB_EAHEAD;  // edge-word lead over the row requests (chunks)

enum { ST_IT1, ST_IT2, ST_E1, ST_E2, ST_U1, ST_U2, ST_F1, ST_F2, ST_IMP, ST_REACH, ST_PREC, ST_S1, ST_S2, ST_T1, ST_T2,
       NSTAT };
enum { CT0 = 8, CTS = 3, CT_LIST = 0, CT_ACTIVE = 1, CT_TILE = 2 };

struct BParams {
    uint32_t n, words, dbits, dmask;
    GraphView G, C;
    const uint32_t* srcs;
    int32_t n_src;
    int two_phase;
    void* out;                  // caller layout: row q of n values in out_fmt (cg_out_format)
    uint32_t* p1;               // nullable, caller layout (u32)
    int out_fmt;
    uint32_t* V;                // [n][RW] value rows
    uint32_t* M;                // [n] active-query masks
    uint32_t* bitmap;           // [words] union frontier
    uint32_t* lv;               // compacted union frontier: vertex, edge offset, query mask
    uint32_t* lo;
    uint32_t* lm;
    unsigned long long* ctrl;   // [0] barrier; [CT0 + CTS*slot + k] per-iteration counters
    unsigned long long* stats;  // nullable: per query NSTAT counters
    uint32_t* err;              // this call's lane-overflow word (ERR_LANE_OVERFLOW)
    uint32_t* err_map;          // the graph's sticky error word (host-mapped): ERR_SOURCE / ERR_ITERS / ERR_NARROW
    const uint32_t* guard;      // non-null: run only if *guard has ERR_LANE_OVERFLOW (the u32-lane re-run)
    uint32_t max_iters;
    uint32_t bits_below;        // frontiers smaller than this keep a bitmap (else the masks M are scanned)
    GraphView R;                // G^R: in-edges for the NEXT-1 pull
    GraphView Rst;              // G minus the CG: phase 2's first sweep (reading N7); ptr null: G
    int dyn;                    // S2's second half in dynamically taken tiles
    const uint32_t* HB;         // CG hub rows [n][2K] for the certificates (nullable; u32 lanes only)
    uint32_t K, KP;             // hubs in HB; row stride 2*KP (KP = K rounded up to a multiple of 4)
    int reduced;                // phase 2 starts with the certificate-driven pull (NEXT-1)
    uint32_t fresh;             // bit p-1: phase p pre-reads values from L2 instead of L1
    // phase-1 pull over CG^R (relax_pull_all): dense iterations
    GraphView RC;               // CG^R (in-edges of the Core Graph)
    const uint32_t* pl_v;       // vertices with CG in-edges (vertex order) ...
    const uint32_t* pl_lo;      // ... and their first in-edge in RC
    uint32_t pl_count, pl_E;    // how many; |E_c|
    uint32_t pl_thr;            // pull a phase-1 iteration whose push would scan >= pl_thr edges (0: never)
    unsigned long long* trace;  // nullable: per iteration {t_start, t_s1, t_s2, phase<<62|q0<<32|listed, active<<32|edges}
    uint32_t trace_cap;
    unsigned long long* trace_cta;  // nullable: per iteration {first, last} CTA S2 finish times
};

// ------------------------------------------------------------------ value lanes
// A row = RW u32 words = Q query lanes, QPW lanes per word.  Per policy:
//   init_word()          every lane InitVal (Alg 3 l.4, l.6)
//   decode(word, j)      lane j in the caller's u32 encoding (Table 6 values; binary32 for Viterbi)
//   live(word)           QPW-bit mask of lanes != InitVal (reached)
//   top(word)            QPW-bit mask of lanes == the lattice top (final by definition)
//   seed(p, j, val)      set lane j of *p (a word holding InitVal there) to the encoded val
//   src_val(), nb_val(w) SourceInitVal and SourceInitVal (+) w, encoded (Alg 3 l.5, l.8)
//   relax(p, uw, cw, w, act, ...)  Process + EdgeFunction of one word (Alg 3 l.22-27): the lanes
//       of act whose candidate ext(uw, w) is better than cw; returns the changed lanes
// RN(1/w) for w = 0..64 (Viterbi's per-edge reciprocal, reading N5): one shared-memory load per edge
// instead of an IEEE-rounded reciprocal sequence; filled by each CTA at kernel start (exact: __frcp_rn)
__shared__ float s_rcp[65];

template <int KIND, int QN>
struct Lanes32 {  // one u32 per query (Table 6 types), QN queries per pass, CGB_G32 words per relax group
    using O = Op<KIND>;
#ifndef CGB_G32
#define CGB_G32 16  // queries per relax group (measured on C2 Viterbi: 4 -> 5.06 ms, 8 -> 4.76, 16 -> 4.65)
#endif
    static constexpr int Q = QN, QPW = 1, RW = QN, G = CGB_G32;
    __device__ static uint32_t init_word() { return O::INIT; }
    __device__ static uint32_t decode(uint32_t x, uint32_t) { return x; }
    __device__ static uint32_t live(uint32_t x) { return x != O::INIT; }
    __device__ static uint32_t top(uint32_t x) { return x == O::SRC; }
    __device__ static void seed(uint32_t* p, uint32_t, uint32_t val) { *p = val; }
    __device__ static uint32_t src_val() { return O::SRC; }
    __device__ static uint32_t nb_val(uint32_t w) { return O::ext(O::SRC, w); }
    static constexpr bool VIT = KIND == CG_VITERBI;
    using Arg = typename std::conditional<VIT, VitArg, uint32_t>::type;  // per-edge, shared by the row
    __device__ static Arg arg(uint32_t w) {
        if constexpr (VIT) return VitArg{w, w <= 64u ? s_rcp[w] : 0.0f};  // RN(1/w) from the CTA's table
        else return w;
    }
    // the pull (phase 1 over CG^R): one query's candidate from u's word, the select of two words
    __device__ static uint32_t cand(uint32_t u, const Arg& w) {
        if (u == O::INIT) return O::INIT;  // an unreached u has no candidate (SSSP / BFS would wrap)
        if constexpr (VIT) return vit_div(u, w);
        else return O::ext(u, w);
    }
    __device__ static uint32_t sel(uint32_t a, uint32_t b) { return O::better(a, b) ? a : b; }
    __device__ static uint32_t improve(uint32_t b, uint32_t c) { return O::better(b, c) ? 1u : 0u; }
    // Process + EdgeFunction of G queries: candidates and Needed tests for all G without
    // branches, then one EdgeFunction per needed query (act: 4 query bits; an unreached u —
    // a pull may read one — is never Needed).
    __device__ static uint32_t relax(uint32_t* p, const uint32_t (&u)[G], const uint32_t (&c)[G], const Arg& w,
                                     uint32_t act, uint32_t& n_edges, uint32_t& n_upd, uint32_t*) {
        uint32_t cand[G], ok = 0, ch = 0;
#pragma unroll
        for (int i = 0; i < G; ++i) ok |= (uint32_t)(u[i] != O::INIT) << i;
        ok &= act;
        n_edges += __popc(ok);
        if constexpr (VIT) {
            vit_div4(u, w, cand);
        } else {
#pragma unroll
            for (int i = 0; i < G; ++i) cand[i] = O::ext(u[i], w);
        }
#pragma unroll
        for (int i = 0; i < G; ++i) ch |= (uint32_t)O::better(cand[i], c[i]) << i;  // Needed(e(u,v))
        ch &= ok;
        if (!ch) return 0u;
#pragma unroll
        for (int i = 0; i < G; ++i)
            if ((ch >> i) & 1u) O::edge_fn(p + i, cand[i]);  // EdgeFunction
        n_upd += __popc(ch);
        return ch;
    }
};

// f16 lanes (binary16 numbers; their bit patterns order like the values because all values
// are >= 0): SSSP / SSNP / BFS: InitVal +inf, SourceInitVal 0, select min; SSWP: InitVal 0,
// SourceInitVal +inf (above every weight), select max.  Integers up to 2048 are exact in
// binary16: SSWP / SSNP values are edge weights (the host requires w_max <= 2048); SSSP / BFS
// raise ERR_LANE_OVERFLOW when a candidate reaches 2048 and the host re-runs the call with u32
// lanes.  The EdgeFunction of 8 lanes is ONE red.min/max.noftz.v4.f16x2 (REDG.F16x8) of a
// 16 B chunk whose non-improving lanes hold the neutral value.  Decoded +inf is 0xFFFFFFFF (SSWP's
// SourceInitVal, the other kinds' InitVal).
template <int KIND>
struct Lanes16 {
    static_assert(KIND == CG_SSSP || KIND == CG_SSWP || KIND == CG_SSNP || KIND == CG_BFS, "f16 lanes");
#ifndef CGB_G16
#define CGB_G16 16  // measured on C2: 4 -> 11.54 K q/s, 8 -> 11.83 K, 16 -> 11.89 K
#endif
    static constexpr int Q = 32, QPW = 2, RW = 16, G = CGB_G16;  // words per relax group (multiple of 4)
    using Arg = uint32_t;
    __device__ static Arg arg(uint32_t w) { return w; }
    static constexpr bool MAXK = KIND == CG_SSWP;
    static constexpr uint32_t INF16 = 0x7c00u, LIMIT = 0x68006800u;  // +inf; 2048.0 in both lanes
    static constexpr uint32_t INIT16 = MAXK ? 0u : INF16, SRC16 = MAXK ? INF16 : 0u;
    __device__ static uint32_t init_word() { return INIT16 * 0x10001u; }
    // lane j as a u32: values are integers in [0, 2048] (or +inf), so the binary16 pattern
    // decodes with integer ops — significand with its hidden bit, times 2, shifted right by
    // 26 - biased exponent (0 -> 0 falls out of the shift; exponent 26 is 2048) — instead of
    // two quarter-rate conversions
    __device__ static uint32_t decode(uint32_t x, uint32_t j) {
        const uint32_t h = (x >> (16 * j)) & 0xffffu;
        const uint32_t k = (((h & 0x3ffu) | 0x400u) << 1) >> min(26u - (h >> 10), 31u);
        return h == INF16 ? 0xffffffffu : k;
    }
    __device__ static uint32_t bits2(uint32_t m) { return ((m >> 15) & 1u) | ((m >> 30) & 2u); }  // 0xffff lanes -> 2 bits
    __device__ static uint32_t halves2(uint32_t b) { return ((b & 1u) ? 0xffffu : 0u) | ((b & 2u) ? 0xffff0000u : 0u); }
    __device__ static uint32_t live(uint32_t x) { return bits2(__vcmpne2(x, init_word())); }
    __device__ static uint32_t top(uint32_t x) { return bits2(__vcmpeq2(x, SRC16 * 0x10001u)); }
    __device__ static void seed(uint32_t* p, uint32_t j, uint32_t val) {  // one writer per (vertex, lane)
        reinterpret_cast<unsigned short*>(p)[j] = (unsigned short)val;
    }
    __device__ static uint32_t src_val() { return SRC16; }
    __device__ static uint32_t h16(uint32_t w) { return __half_as_ushort(__uint2half_rn(w)); }
    __device__ static uint32_t nb_val(uint32_t w) { return KIND == CG_BFS ? 0x3c00u : h16(w); }
    __device__ static uint32_t ext2(uint32_t u, uint32_t w2) {
        const __half2 a = *reinterpret_cast<const __half2*>(&u), b = *reinterpret_cast<const __half2*>(&w2);
        __half2 r;
        if (KIND == CG_SSWP) r = __hmin2(a, b);
        else if (KIND == CG_SSNP) r = __hmax2(a, b);
        else r = __hadd2(a, b);  // SSSP: + w; BFS: + 1
        return *reinterpret_cast<const uint32_t*>(&r);
    }
    __device__ static uint32_t needed2(uint32_t x, uint32_t c) {  // 0xffff per lane whose candidate is better
        const __half2 a = *reinterpret_cast<const __half2*>(&x), b = *reinterpret_cast<const __half2*>(&c);
        return MAXK ? __hgt2_mask(a, b) : __hlt2_mask(a, b);
    }
    __device__ static uint32_t sel2(uint32_t x, uint32_t c) {  // the better of two words, per lane
        const __half2 a = *reinterpret_cast<const __half2*>(&x), b = *reinterpret_cast<const __half2*>(&c);
        const __half2 r = MAXK ? __hmax2(a, b) : __hmin2(a, b);
        return *reinterpret_cast<const uint32_t*>(&r);
    }
    // the pull (phase 1 over CG^R): the candidates of u's word (+inf stays +inf), per-lane select
    __device__ static uint32_t cand(uint32_t u, Arg w) { return ext2(u, (KIND == CG_BFS ? 0x3c00u : h16(w)) * 0x10001u); }
    __device__ static uint32_t sel(uint32_t a, uint32_t b) { return sel2(a, b); }
    __device__ static uint32_t improve(uint32_t b, uint32_t c) { return bits2(needed2(b, c)); }
    __device__ static bool overflow(uint32_t b, uint32_t c) {  // an improving lane reached 2048 (SSSP / BFS)
        return (KIND == CG_SSSP || KIND == CG_BFS) && (__vcmpgeu2(b, LIMIT) & needed2(b, c)) != 0u;
    }
    // Process + EdgeFunction of one 16 B chunk (4 words, 8 queries); act: 8 query bits.
    // The Needed test is taken on every lane, not only the active ones: a lane whose u is not
    // active for its query holds a value already pushed along (u, v), so its candidate is never
    // better than Val(v) — except against a stale pre-read, where applying it is still a valid
    // relaxation (a real path value) and v becomes active for that query (reading N1).  The
    // EdgeFunction therefore sends the candidates themselves: a non-needed lane's candidate is no
    // better than the current Val(v) and leaves it unchanged.  Common case (nothing needed): one
    // packed ⊕, one packed compare and an OR per word.
    __device__ static uint32_t relax(uint32_t* p, const uint32_t (&u)[G], const uint32_t (&c)[G], Arg w,
                                     uint32_t act, uint32_t& n_edges, uint32_t& n_upd, uint32_t* err) {
        if (!act) return 0u;
        n_edges += __popc(act);
        const uint32_t w2 = (KIND == CG_BFS ? 0x3c00u : h16(w)) * 0x10001u;
        uint32_t x[G], bm[G], any = 0;
#pragma unroll
        for (int i = 0; i < G; ++i) {
            x[i] = ext2(u[i], w2);
            bm[i] = needed2(x[i], c[i]);
            any |= bm[i];
        }
        if (!any) return 0u;
        uint32_t ch = 0, over = 0;
#pragma unroll
        for (int i = 0; i < G; ++i) {
            if (KIND == CG_SSSP || KIND == CG_BFS) over |= __vcmpgeu2(x[i], LIMIT) & bm[i];
            ch |= bits2(bm[i]) << (2 * i);
        }
        if (over) atomicOr(err, ERR_LANE_OVERFLOW);
#pragma unroll
        for (int h = 0; h < G / 4; ++h) {  // one 16 B vector EdgeFunction per 8 queries with a needed lane
            if (!((ch >> (8 * h)) & 0xffu)) continue;
            if (MAXK)
                asm volatile("red.relaxed.gpu.global.max.noftz.v4.f16x2 [%0], {%1,%2,%3,%4};" ::"l"(p + 4 * h),
                             "r"(x[4 * h]), "r"(x[4 * h + 1]), "r"(x[4 * h + 2]), "r"(x[4 * h + 3])
                             : "memory");
            else
                asm volatile("red.relaxed.gpu.global.min.noftz.v4.f16x2 [%0], {%1,%2,%3,%4};" ::"l"(p + 4 * h),
                             "r"(x[4 * h]), "r"(x[4 * h + 1]), "r"(x[4 * h + 2]), "r"(x[4 * h + 3])
                             : "memory");
        }
        n_upd += __popc(ch);
        return ch;
    }
};

// one bit per query (REACH): InitVal 0, SourceInitVal 1, cand = u; EdgeFunction red.or
struct LanesBit {
    static constexpr int Q = 32, QPW = 32, RW = 1, G = 1;
    using Arg = uint32_t;
    __device__ static Arg arg(uint32_t w) { return w; }
    __device__ static uint32_t init_word() { return 0u; }
    __device__ static uint32_t decode(uint32_t x, uint32_t j) { return (x >> j) & 1u; }
    __device__ static uint32_t live(uint32_t x) { return x; }
    __device__ static uint32_t top(uint32_t x) { return x; }
    __device__ static void seed(uint32_t* p, uint32_t j, uint32_t) { atomicOr(p, 1u << j); }
    __device__ static uint32_t src_val() { return 1u; }
    __device__ static uint32_t nb_val(uint32_t) { return 1u; }
    __device__ static uint32_t cand(uint32_t u, uint32_t) { return u; }
    __device__ static uint32_t sel(uint32_t a, uint32_t b) { return a | b; }
    __device__ static uint32_t improve(uint32_t b, uint32_t c) { return b & ~c; }
    __device__ static uint32_t relax(uint32_t* p, const uint32_t (&u)[G], const uint32_t (&c)[G], uint32_t,
                                     uint32_t act, uint32_t& n_edges, uint32_t& n_upd, uint32_t*) {
        n_edges += __popc(act);
        const uint32_t nw = u[0] & act & ~c[0];  // Needed: u reached, v not
        if (!nw) return 0u;
        red_or(p, nw);
        n_upd += __popc(nw);
        return nw;
    }
};

// WCC (NEXT-3; Table 6 WCC row): one label per vertex, Val(v) = v initially, every vertex
// active at the start of both phases (reading W2), cand = Val(u), select min (red.min).
struct LanesLabel {
    static constexpr int Q = 1, QPW = 1, RW = 1, G = 1;
    using Arg = uint32_t;
    __device__ static Arg arg(uint32_t w) { return w; }
    static constexpr bool ALL_ACTIVE = true;
    __device__ static uint32_t init_word() { return 0xffffffffu; }  // (never a label: the stats' "unreached")
    __device__ static uint32_t init_at(uint64_t i) { return (uint32_t)i; }
    __device__ static uint32_t decode(uint32_t x, uint32_t) { return x; }
    __device__ static uint32_t live(uint32_t) { return 1u; }
    __device__ static uint32_t top(uint32_t) { return 0u; }
    __device__ static void seed(uint32_t*, uint32_t, uint32_t) {}
    __device__ static uint32_t src_val() { return 0u; }
    __device__ static uint32_t nb_val(uint32_t) { return 0u; }
    __device__ static uint32_t relax(uint32_t* p, const uint32_t (&u)[G], const uint32_t (&c)[G], uint32_t,
                                     uint32_t act, uint32_t& n_edges, uint32_t& n_upd, uint32_t*) {
        if (!act) return 0u;
        ++n_edges;
        if (u[0] >= c[0]) return 0u;  // Needed: Val(v) > Val(u)
        red_min(p, u[0]);             // CASMIN(Val(v), Val(u))
        ++n_upd;
        return 1u;
    }
};

// per-vertex initial word and "every vertex starts active" for the policies that need them
template <class L, class = void> struct InitOf {
    static constexpr bool ALL_ACTIVE = false;
    __device__ static uint32_t at(uint64_t) { return L::init_word(); }
};
template <class L> struct InitOf<L, decltype((void)L::ALL_ACTIVE, void())> {
    static constexpr bool ALL_ACTIVE = L::ALL_ACTIVE;
    __device__ static uint32_t at(uint64_t i) { return L::init_at(i); }
};

template <int LW, int KIND> struct LanesOf;
template <int KIND> struct LanesOf<2, KIND> { using T = LanesLabel; };
template <int KIND> struct LanesOf<32, KIND> { using T = Lanes32<KIND, 16>; };  // u32 fallback: 16 per pass
template <int KIND> struct LanesOf<33, KIND> { using T = Lanes32<KIND, 32>; };  // Viterbi: 32 per pass (128 B rows)
template <int KIND> struct LanesOf<16, KIND> { using T = Lanes16<KIND>; };
template <int KIND> struct LanesOf<1, KIND> { using T = LanesBit; };

template <class L>
__device__ __forceinline__ uint32_t group_mask(uint32_t mask, int i) {  // the lanes of word group i in a query mask
    constexpr int LG = L::QPW * L::G;  // lanes per relax group
    return LG >= 32 ? mask : (mask >> (i * LG)) & ((1u << LG) - 1u);
}

// queries with a non-InitVal value at v (L2 reads: values other SMs update; 16 B vector loads)
template <class L>
__device__ __forceinline__ uint32_t row_live(const uint32_t* V, uint32_t v) {
    const uint32_t* r = V + (size_t)v * L::RW;
    uint32_t m = 0;
    if constexpr (L::RW % 4 == 0) {
#pragma unroll
        for (int i = 0; i < L::RW / 4; ++i) {
            uint4 x;
            asm volatile("ld.global.cg.v4.u32 {%0,%1,%2,%3}, [%4];"
                         : "=r"(x.x), "=r"(x.y), "=r"(x.z), "=r"(x.w)
                         : "l"(reinterpret_cast<const uint4*>(r) + i));
            m |= (L::live(x.x) | L::live(x.y) << L::QPW | L::live(x.z) << (2 * L::QPW) | L::live(x.w) << (3 * L::QPW))
                 << (4 * i * L::QPW);
        }
    } else {
#pragma unroll
        for (int i = 0; i < L::RW; ++i) m |= L::live(ld_cg(r + i)) << (i * L::QPW);
    }
    return m;
}

// ------------------------------------------------------------------ NEXT-1 certificates
// p = Val(s,v) after phase 1 on the CG, a bound on the true value from the "worse" side.
// Fv/Rv = Q(h) on G / on G^R at v, Fs/Rs the same at the source.  A certificate is a bound
// from the other side, met with equality (Theorem 1; bottleneck analogs):
//   SSWP (p <= W(s,v)): W(v,h) > W(s,h) => W(s,v) <= W(s,h);  W(h,s) > W(h,v) => W(s,v) <= W(h,v)
//   SSNP (p >= N(s,v)): N(v,h) < N(s,h) => N(s,v) >= N(s,h);  N(h,s) < N(h,v) => N(s,v) >= N(h,v)
//   SSSP (p >= d(s,v)): d(s,v) >= d(s,h) - d(v,h);  d(s,v) >= d(h,v) - d(h,s)  (Theorem 1), with
//        "infinite minus finite" = infinite (s cannot reach v when v reaches h but s does not, ...)
template <int KIND>
__device__ __forceinline__ bool certified(uint32_t p, uint32_t Fv, uint32_t Rv, uint32_t Fs, uint32_t Rs) {
    if (KIND == CG_SSWP) return (Rv > Rs && p == Rs) || (Fs > Fv && p == Fv);
    if (KIND == CG_SSNP) return (Rv < Rs && p == Rs) || (Fs < Fv && p == Fv);
    if (KIND == CG_SSSP) {
        constexpr uint32_t INF = 0xffffffffu;
        if (Rv != INF && p == (Rs == INF ? INF : (Rs > Rv ? Rs - Rv : 0u))) return true;
        if (Fs != INF && p == (Fv == INF ? INF : (Fv > Fs ? Fv - Fs : 0u))) return true;
    }
    return false;
}

// queries q < nq whose phase-1 value at v is not proven final (Reduced(E) keeps v's in-edges):
// the lattice top is final (REACH: reached); u32 lanes may add the hub certificates.  Kept
// register-light (it runs inside the persistent kernel).
template <int KIND, class L>
__device__ uint32_t uncertified(const BParams& P, const uint32_t* sh, int nq, uint32_t v) {
    constexpr uint32_t WM = L::QPW == 32 ? 0xffffffffu : (1u << L::QPW) - 1u;
    const uint32_t* row = P.V + (size_t)v * L::RW;
    uint32_t unc = 0;
#pragma unroll
    for (int i = 0; i < L::RW; ++i) unc |= (~L::top(ld_cg(row + i)) & WM) << (i * L::QPW);
    unc &= nq >= 32 ? 0xffffffffu : ((1u << nq) - 1u);
    if (L::QPW != 1 || KIND == CG_REACH || P.HB == nullptr || !unc) return unc;
    // hub row of v: F at [0, KP), R at [KP, 2 KP) (KP = K rounded up to 4: 16 B aligned chunks)
    const uint32_t K = P.K, KP = P.KP;
    const uint4* hb = reinterpret_cast<const uint4*>(P.HB + (size_t)v * 2 * KP);
    uint32_t todo = unc;
    while (todo) {
        const int q = __ffs(todo) - 1;
        todo &= todo - 1;
        const uint32_t p = ld_cg(row + q);
        const uint32_t* sq = sh + q * 2 * K;
        for (uint32_t h0 = 0; h0 < K; h0 += 4) {
            const uint4 f = __ldg(hb + h0 / 4), r = __ldg(hb + (KP + h0) / 4);
            bool c = false;
#pragma unroll
            for (int j = 0; j < 4; ++j) {
                const uint32_t h = h0 + j;
                const uint32_t Fv = j == 0 ? f.x : j == 1 ? f.y : j == 2 ? f.z : f.w;
                const uint32_t Rv = j == 0 ? r.x : j == 1 ? r.y : j == 2 ? r.z : r.w;
                c |= h < K && certified<KIND>(p, Fv, Rv, sq[h], sq[K + h]);
            }
            if (c) {
                unc &= ~(1u << q);
                break;
            }
        }
    }
    return unc;
}

// ------------------------------------------------------------------ S1 (union frontier)
// S1 modes: F_BITS (small frontiers: bitmap bits set by S2), F_MASKS (frontier = {v : M[v] != 0}),
// F_IMPACTED (Alg 3 l.15: v active for q iff Val(v) != InitVal), F_UNCERT (NEXT-1: v active for
// its uncertified queries; degrees are then in-degrees, g = G^R).  compact_bits (F_BITS): pass 1
// counts the active vertices with edges and their edges per warp and reserves the CTA's list
// range with ONE 64-bit atomicAdd; pass 2 writes (v, edge offset, query mask) in vertex order,
// consuming the masks and the bitmap bits.
enum { F_BITS = 0, F_MASKS = 1, F_IMPACTED = 2, F_UNCERT = 3 };

__device__ void compact_bits(const BParams& P, const GraphView& g, unsigned long long* cnt_slot,
                             unsigned long long* act_slot, uint32_t* sm) {
    const uint32_t lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const uint64_t W = P.words;
    const uint32_t w0 = (uint32_t)(W * blockIdx.x / gridDim.x), w1 = (uint32_t)(W * (blockIdx.x + 1) / gridDim.x);
    const uint32_t lt = (1u << lane) - 1u;

    uint32_t cnt = 0, edges = 0, active = 0;
    for (uint32_t g0 = w0 + warp * 32; g0 < w1; g0 += BW * 32) {
        const uint32_t wi = g0 + lane;
        uint32_t word = 0;
        if (wi < w1) word = ld_cg(P.bitmap + wi);
        active += __popc(word);
        uint32_t nz = __ballot_sync(FULL, word != 0);
        while (nz) {
            int js[CW];
            uint32_t deg[CW];
            word_degrees(g, P.n, g0, nz, lane, js, deg);
#pragma unroll
            for (int k = 0; k < CW; ++k) {
                if (js[k] < 0) break;
                if ((__shfl_sync(FULL, word, js[k]) >> lane) & 1u) {
                    cnt += deg[k] != 0;
                    edges += deg[k];
                }
            }
        }
    }
    for (int o = 16; o > 0; o >>= 1) {
        cnt += __shfl_xor_sync(FULL, cnt, o);
        edges += __shfl_xor_sync(FULL, edges, o);
        active += __shfl_xor_sync(FULL, active, o);
    }
    if (lane == 0) {
        sm[warp] = cnt;
        sm[BW + warp] = edges;
        if (active) atomicAdd(act_slot, (unsigned long long)active);
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        uint32_t tc = 0, te = 0;
        for (int i = 0; i < BW; ++i) {
            const uint32_t c = sm[i], e = sm[BW + i];
            sm[i] = tc;
            sm[BW + i] = te;
            tc += c;
            te += e;
        }
        unsigned long long old = 0;
        if (tc) old = atomicAdd(cnt_slot, ((unsigned long long)tc << 32) | te);
        sm[2 * BW] = (uint32_t)(old >> 32);
        sm[2 * BW + 1] = (uint32_t)old;
    }
    __syncthreads();
    uint32_t pos = sm[2 * BW] + sm[warp];
    uint32_t eb = sm[2 * BW + 1] + sm[BW + warp];
    __syncthreads();

    for (uint32_t g0 = w0 + warp * 32; g0 < w1; g0 += BW * 32) {
        const uint32_t wi = g0 + lane;
        const uint32_t word = (wi < w1) ? ld_cg(P.bitmap + wi) : 0u;
        if (word) P.bitmap[wi] = 0u;
        uint32_t nz = __ballot_sync(FULL, word != 0);
        while (nz) {
            int js[CW];
            uint32_t deg[CW];
            word_degrees(g, P.n, g0, nz, lane, js, deg);
#pragma unroll
            for (int k = 0; k < CW; ++k) {
                if (js[k] < 0) break;
                const uint32_t v = (g0 + js[k]) * 32 + lane;
                const bool act = (__shfl_sync(FULL, word, js[k]) >> lane) & 1u;
                const uint32_t d = act ? deg[k] : 0u;
                uint32_t mask = 0;
                if (act) {
                    mask = ld_cg(P.M + v);
                    P.M[v] = 0u;  // consumed
                }
                uint32_t incl = d;
#pragma unroll
                for (int o = 1; o < 32; o <<= 1) {
                    const uint32_t y = __shfl_up_sync(FULL, incl, o);
                    if (lane >= (uint32_t)o) incl += y;
                }
                const uint32_t bal = __ballot_sync(FULL, d != 0);
                if (d) {
                    const uint32_t i = pos + __popc(bal & lt);
                    P.lv[i] = v;
                    P.lo[i] = eb + incl - d;
                    P.lm[i] = mask;
                }
                pos += __popc(bal);
                eb += __shfl_sync(FULL, incl, 31);
            }
        }
    }
}

#ifndef CGB_S1_SPARSE
#define CGB_S1_SPARSE 1  // S1 reads row bounds only for vertices with a nonzero mask
#endif
// S1 for large frontiers held as query masks M (F_MASKS, and F_IMPACTED / F_UNCERT after their
// mark pass): no bitmap.  A warp issues the masks and row offsets of 16 bitmap words (512
// vertices) at once — one memory round trip instead of a dependent degree fetch per active word.
__device__ __forceinline__ void span_loads(const BParams& P, const GraphView& g, uint32_t g0, uint32_t w1, int h,
                                           uint32_t (&mv)[16], uint32_t (&dg)[16]) {
    const uint32_t lane = threadIdx.x & 31;
    uint32_t pv[16];
#if CGB_S1_SPARSE
    // masks first, then the row bounds of the active vertices only: sparse frontiers (most
    // iterations) read M alone instead of M + two offset arrays
#pragma unroll
    for (int j = 0; j < 16; ++j) {
        const uint32_t wj = g0 + h * 16 + j;
        const uint32_t v = wj * 32 + lane;
        mv[j] = (wj < w1 && v < P.n) ? ld_cg(P.M + v) : 0u;
    }
    const uint32_t* pe = g.end ? g.end : g.ptr + 1;
#pragma unroll
    for (int j = 0; j < 16; ++j) {
        const uint32_t v = (g0 + h * 16 + j) * 32 + lane;
        pv[j] = mv[j] ? __ldg(g.ptr + v) : 0u;
        dg[j] = mv[j] ? __ldg(pe + v) : 0u;
    }
#pragma unroll
    for (int j = 0; j < 16; ++j) dg[j] -= pv[j];
    return;
#endif
    if (g.end) {  // split rows: [ptr[v], end[v])
#pragma unroll
        for (int j = 0; j < 16; ++j) {
            const uint32_t wj = g0 + h * 16 + j;
            const uint32_t v = wj * 32 + lane;
            const bool ok = wj < w1 && v < P.n;
            mv[j] = ok ? ld_cg(P.M + v) : 0u;
            pv[j] = ok ? __ldg(g.ptr + v) : 0u;
            dg[j] = ok ? __ldg(g.end + v) : 0u;
        }
#pragma unroll
        for (int j = 0; j < 16; ++j) dg[j] = mv[j] ? dg[j] - pv[j] : 0u;
        return;
    }
#pragma unroll
    for (int j = 0; j < 16; ++j) {
        const uint32_t wj = g0 + h * 16 + j;
        const uint32_t v = wj * 32 + lane;
        const bool ok = wj < w1 && v < P.n;
        mv[j] = ok ? ld_cg(P.M + v) : 0u;
        pv[j] = __ldg(g.ptr + min(v, P.n));
    }
    const uint32_t pn = __ldg(g.ptr + min((g0 + h * 16 + 16) * 32, P.n));  // row offset after the span
#pragma unroll
    for (int j = 0; j < 16; ++j) {
        uint32_t nx = __shfl_down_sync(FULL, pv[j], 1);
        const uint32_t n31 = j < 15 ? __shfl_sync(FULL, pv[j < 15 ? j + 1 : j], 0) : pn;
        if (lane == 31) nx = n31;
        dg[j] = mv[j] ? nx - pv[j] : 0u;
    }
}

#ifndef CGB_S1H
#define CGB_S1H 2
#endif
__device__ void compact_masks(const BParams& P, const GraphView& g, unsigned long long* cnt_slot,
                              unsigned long long* act_slot, uint32_t* sm) {
    // One pass: the CTA's word range is taken in rounds of BW x H half-spans (H x 16 words =
    // H x 512 vertices per warp, all loads of a round issued together); a round's masks and
    // degrees stay in registers while the CTA reserves its list range (one 64-bit atomicAdd
    // per round), then the entries are written and the masks consumed.  List order is vertex
    // order within a round; S2 needs only that the edge offsets ascend with the list index,
    // which the packed (count, edges) reservation gives.
    constexpr int H = CGB_S1H;
    const uint32_t lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const uint64_t W = P.words;
    const uint32_t w0 = (uint32_t)(W * blockIdx.x / gridDim.x), w1 = (uint32_t)(W * (blockIdx.x + 1) / gridDim.x);
    const uint32_t lt = (1u << lane) - 1u;
    uint32_t active = 0;
    for (uint32_t r0 = w0; r0 < w1; r0 += BW * 16 * H) {
        const uint32_t g0 = r0 + warp * 16 * H;
        uint32_t mv[H][16], dg[H][16];
#pragma unroll
        for (int h = 0; h < H; ++h) span_loads(P, g, g0, w1, h, mv[h], dg[h]);
        uint32_t cnt = 0, edges = 0;
#pragma unroll
        for (int h = 0; h < H; ++h)
#pragma unroll
            for (int j = 0; j < 16; ++j) {
                active += mv[h][j] != 0u;
                cnt += dg[h][j] != 0u;
                edges += dg[h][j];
            }
        for (int o = 16; o > 0; o >>= 1) {
            cnt += __shfl_xor_sync(FULL, cnt, o);
            edges += __shfl_xor_sync(FULL, edges, o);
        }
        if (lane == 0) {
            sm[warp] = cnt;
            sm[BW + warp] = edges;
        }
        __syncthreads();
        if (threadIdx.x == 0) {
            uint32_t tc = 0, te = 0;
            for (int i = 0; i < BW; ++i) {
                const uint32_t c = sm[i], e = sm[BW + i];
                sm[i] = tc;
                sm[BW + i] = te;
                tc += c;
                te += e;
            }
            unsigned long long old = 0;
            if (tc) old = atomicAdd(cnt_slot, ((unsigned long long)tc << 32) | te);
            sm[2 * BW] = (uint32_t)(old >> 32);
            sm[2 * BW + 1] = (uint32_t)old;
        }
        __syncthreads();
        uint32_t pos = sm[2 * BW] + sm[warp];
        uint32_t eb = sm[2 * BW + 1] + sm[BW + warp];
        __syncthreads();  // sm is rewritten by the next round
#pragma unroll
        for (int h = 0; h < H; ++h)
#pragma unroll
            for (int j = 0; j < 16; ++j) {
                const uint32_t v = (g0 + h * 16 + j) * 32 + lane;
                if (mv[h][j]) P.M[v] = 0u;  // consumed
                const uint32_t d = dg[h][j];
                uint32_t incl = d;
#pragma unroll
                for (int o = 1; o < 32; o <<= 1) {
                    const uint32_t y = __shfl_up_sync(FULL, incl, o);
                    if (lane >= (uint32_t)o) incl += y;
                }
                const uint32_t bal = __ballot_sync(FULL, d != 0);
                if (d) {
                    const uint32_t i = pos + __popc(bal & lt);
                    P.lv[i] = v;
                    P.lo[i] = eb + incl - d;
                    P.lm[i] = mv[h][j];
                }
                pos += __popc(bal);
                eb += __shfl_sync(FULL, incl, 31);
            }
    }
    for (int o = 16; o > 0; o >>= 1) active += __shfl_xor_sync(FULL, active, o);
    if (lane == 0 && active) atomicAdd(act_slot, (unsigned long long)active);
}

// Mark passes (thread per vertex, coalesced): F_IMPACTED — Alg 3 l.15, M[v] = the queries for
// which Val(v) != InitVal; F_UNCERT — NEXT-1, M[v] = v's uncertified queries, only for vertices
// with in-edges (the pull needs them).  M is all-zero before either.
template <int KIND, class L>
__device__ void mark_masks(const BParams& P, int mode, const uint32_t* sh, int nq) {
    const uint64_t nth = (uint64_t)gridDim.x * BT;
    for (uint64_t v = blockIdx.x * (uint64_t)BT + threadIdx.x; v < P.n; v += nth) {
        uint32_t m;
        if (mode == F_IMPACTED) m = row_live<L>(P.V, (uint32_t)v);
        else m = __ldg(P.R.ptr + v + 1) > __ldg(P.R.ptr + v) ? uncertified<KIND, L>(P, sh, nq, (uint32_t)v) : 0u;
        if (m) P.M[v] = m;
    }
}

// ------------------------------------------------------------------ S2 (lane = edge, row over queries)
// Bytes of one (<= 16 B) cp.async copy of a row, copies per row, and the XOR swizzle of a lane's
// row in a pipeline stage: copy i of lane L's row sits at slot i ^ sw(L), so the 32 lanes'
// shared-memory reads of word w hit all banks.
template <class L> struct RowCopy {
    static constexpr uint32_t CB = L::RW >= 4 ? 16u : 4u * L::RW;  // bytes per copy
    static constexpr uint32_t CW4 = CB / 4;                         // words per copy
    static constexpr uint32_t C = L::RW / CW4;                      // copies per row
    static constexpr uint32_t LPL = 4 * L::RW >= 128 ? 1u : 128u / (4 * L::RW);  // lanes per 128 B
    __device__ static uint32_t sw(uint32_t lane) { return C > 1 ? (lane / LPL) % C : 0u; }
    __device__ static void copy(uint32_t* dst, const uint32_t* src, bool fresh) {
        if (CB == 16) {
            if (fresh) cp_async16_cg(dst, src);  // Needed pre-read from L2
            else cp_async16_ca(dst, src);        // from L1 (a stale value is never better)
        } else {
            asm volatile("cp.async.ca.shared.global [%0], [%1], %2;" ::"r"(smem_u32(dst)), "l"(src), "n"(CB) : "memory");
        }
    }
};

#ifndef CGB_EDGE_SMEM
#define CGB_EDGE_SMEM 2  // S2's edge words through a shared-memory ring (window_edges_sm): 0 never, 1 every
                         // lane type, 2 one-word rows only (REACH bits, WCC labels; measured on C2: REACH
                         // FULL 1.82 -> 1.54 ms, WCC 1.84 -> 1.53 ms; 64 B rows 2-5 % slower, and slower
                         // still with a deeper row pipeline: profiles/r2_s2_experiments.txt)
#endif
template <class L>
constexpr bool edge_smem() { return CGB_EDGE_SMEM == 1 || (CGB_EDGE_SMEM == 2 && L::RW == 1); }
// edge-word lead over the row requests (chunks): binary16 rows (the cheapest relax per edge) keep
// the edge stream 2 x S_PIPE chunks ahead by default; the u32 rows' heavier relax needs the registers
#ifndef CGB_EA16
#define CGB_EA16 (2 * CGB_STAGES)
#endif
template <class L>
constexpr int ea_lead() { return (L::QPW == 2 && E_AHEAD == S_PIPE) ? CGB_EA16 : E_AHEAD; }

// The edges [e, ehi) of one 32-row window: lane r of the window holds row r's first edge index
// `off`, its address base (edge address = base + edge index) and its query mask; the rows'
// values are in xs (r * RW + word).  Lane L takes edge L of each 32-edge chunk for all Q queries.
// Software pipeline (per-warp ring `vs` of S_PIPE value-row stages in shared memory; E_AHEAD
// edge-word slots in registers): while chunk c is consumed, chunk c + S - 1's value rows are
// requested (cp.async global -> shared) and the edge words of chunk c + S - 1 + E_AHEAD are
// loaded — the edge stream runs E_AHEAD chunks ahead of the row gathers it feeds.
template <int KIND, bool PACKED, class L>
__device__ __forceinline__ void window_edges(const BParams& P, const GraphView& g, const uint32_t* xs, uint32_t* vs,
                                             uint32_t off, uint32_t base, uint32_t mask, uint32_t e, uint32_t ehi,
                                             bool set_bits, bool fresh, uint32_t& n_edges, uint32_t& n_upd,
                                             uint32_t& n_read) {
    constexpr int EA = ea_lead<L>();
    constexpr int S = S_PIPE, RW = L::RW;
    static_assert(EA % S == 0 && EA >= S, "E_AHEAD must be a multiple of S_PIPE");
    using RC = RowCopy<L>;
    constexpr uint32_t NONE = 0xffffffffu;
    const uint32_t lane = threadIdx.x & 31;
    const uint32_t swz = RC::sw(lane);
    if (e >= ehi) return;
    const uint32_t nch = (ehi - e + 31) >> 5;

    EdgeWord<PACKED> ew[EA];       // fetched edge words (slot = chunk % EA)
    uint32_t ek[EA];               // their window row (NONE: no edge / inactive row)
    // requested chunks (slot = chunk % S): destination, weight, window row of each lane's edge —
    // kept in the warp's shared metadata ring (lane-private words), not in registers, so the
    // row pipeline can be deeper without spilling
    uint32_t* const mt = vs + S * 32 * RW;
    auto sd = [&](int slot) -> uint32_t& { return mt[(3 * slot + 0) * 32 + lane]; };
    auto sw = [&](int slot) -> uint32_t& { return mt[(3 * slot + 1) * 32 + lane]; };
    auto sk = [&](int slot) -> uint32_t& { return mt[(3 * slot + 2) * 32 + lane]; };

    // the window row of each lane's edge t = cs + lane: rows starting at or before cs (one
    // ballot) plus the rows starting in (cs, t] (one warp OR of start bits) — no dependent
    // shuffle search; the list holds rows with edges only, so row starts are distinct
    auto fetch = [&](uint32_t c, EdgeWord<PACKED>& wd, uint32_t& kout) {
        const uint32_t cs = e + c * 32, t = cs + lane;
        const uint32_t below = __popc(__ballot_sync(FULL, off <= cs));  // >= 1: row 0 starts at or before e
        const uint32_t rel = off - cs;
        const uint32_t starts = __reduce_or_sync(FULL, (rel - 1u < 31u) ? (1u << rel) : 0u);
        const uint32_t kk = below - 1u + __popc(starts & ((2u << lane) - 1u));
        const uint32_t mk = __shfl_sync(FULL, mask, kk);
        const uint32_t a = __shfl_sync(FULL, base, kk) + t;
        const bool ok = t < ehi && mk != 0u;
        if (ok) wd.load(g, a);
        kout = ok ? kk : NONE;
    };
    // Rows of C > 1 copies are gathered cooperatively: copy instruction i moves piece (lane % C)
    // of the row of lane i * (32 / C) + lane / C, so one instruction touches 32 / C rows of
    // contiguous 16 B pieces instead of 32 scattered lines (C times fewer L1 tag lookups per
    // chunk).  The slot is shared across lanes, so the caller brackets it with __syncwarp().
    auto request = [&](int slot, const EdgeWord<PACKED>& wd, uint32_t kk) {
        sk(slot) = kk;
        uint32_t dd = NONE;
        if (kk != NONE) {
            uint32_t d, w;
            wd.decode(P.dbits, P.dmask, d, w);
            sd(slot) = d;
            sw(slot) = w;
            dd = d;
        }
        if constexpr (RC::C > 1) {
            constexpr uint32_t RPI = 32 / RC::C;  // rows per copy instruction
            const uint32_t p = lane % RC::C;
#pragma unroll
            for (uint32_t i = 0; i < RC::C; ++i) {
                const uint32_t r = i * RPI + lane / RC::C;
                const uint32_t dr = __shfl_sync(FULL, dd, r);
                if (dr != NONE)
                    RC::copy(vs + (slot * 32 + r) * RW + RC::CW4 * (p ^ RC::sw(r)), P.V + (size_t)dr * RW + RC::CW4 * p,
                             fresh);
            }
        } else if (dd != NONE) {
            RC::copy(vs + (slot * 32 + lane) * RW, P.V + (size_t)dd * RW, fresh);
        }
        cp_async_commit();
    };

#pragma unroll
    for (int s = 0; s < EA; ++s) {
        ek[s] = NONE;
        if ((uint32_t)s < nch) fetch(s, ew[s], ek[s]);
    }
#pragma unroll
    for (int s = 0; s < S - 1; ++s) {
        request(s, ew[s], ek[s]);
        ek[s] = NONE;
        if ((uint32_t)(s + EA) < nch) fetch(s + EA, ew[s], ek[s]);
    }
    for (uint32_t c0 = 0; c0 < nch; c0 += EA) {
#pragma unroll
        for (int s = 0; s < EA; ++s) {
            const uint32_t cc = c0 + s;
            if (cc >= nch) break;
            const int je = (s + S - 1) % EA;  // edge slot of chunk cc + S - 1
            const int jr = (s + S - 1) % S;   // its row slot
            if constexpr (RC::C > 1) __syncwarp();  // every lane is done with slot jr (chunk cc - 1)
            request(jr, ew[je], ek[je]);
            ek[je] = NONE;
            if (cc + S - 1 + EA < nch) fetch(cc + S - 1 + EA, ew[je], ek[je]);
            cp_async_wait<S - 1>();  // chunk cc's row pieces this lane copied have landed
            if constexpr (RC::C > 1) __syncwarp();  // ... and those the other lanes copied
            const int sr = s % S;    // chunk cc's row slot
            const uint32_t kk = sk(sr);
            const uint32_t mk = __shfl_sync(FULL, mask, kk & 31u);
            if (kk == NONE) continue;
            ++n_read;
            const uint32_t d = sd(sr);
            const typename L::Arg w = L::arg(sw(sr));         // per edge, shared by the row's queries
            const uint32_t* rv = vs + (sr * 32 + lane) * RW;  // v's row (swizzled copies)
            const uint32_t* ru = xs + kk * RW;               // u's row
            uint32_t* pv = P.V + (size_t)d * RW;
            uint32_t changed = 0;
#pragma unroll
            for (int gi = 0; gi < RW / L::G; ++gi) {
                const uint32_t act = group_mask<L>(mk, gi);
                if (!act) continue;
                uint32_t uu[L::G], cc2[L::G];
#pragma unroll
                for (int j = 0; j < L::G; ++j) {
                    const uint32_t i = (uint32_t)(gi * L::G + j);
                    uu[j] = ru[i];
                    cc2[j] = rv[((i / RC::CW4) ^ swz) * RC::CW4 + i % RC::CW4];
                }
                changed |= L::relax(pv + gi * L::G, uu, cc2, w, act, n_edges, n_upd, P.err) << (gi * L::G * L::QPW);
            }
            if (changed) {
                red_or(P.M + d, changed);                                 // v active for those queries
                if (set_bits) red_or(P.bitmap + (d >> 5), 1u << (d & 31));  // union frontier bit
            }
        }
    }
    cp_async_wait<0>();
}

// window_edges with the edge stream in shared memory as well: edge words are copied (cp.async, 4 or
// 8 B per lane) into a per-warp ring LE = S_PIPE chunks ahead of the row requests, their window rows
// into a lane-private ring beside it — no pipeline state in registers, so the row pipeline can be
// deeper.  One cp.async group per chunk: {rows of chunk c + S - 1, edge words of chunk c + 2S - 1}.
template <int KIND, bool PACKED, class L>
__device__ __forceinline__ void window_edges_sm(const BParams& P, const GraphView& g, const uint32_t* xs,
                                                uint32_t* vs, uint32_t off, uint32_t base, uint32_t mask, uint32_t e,
                                                uint32_t ehi, bool set_bits, bool fresh, uint32_t& n_edges,
                                                uint32_t& n_upd, uint32_t& n_read) {
    constexpr uint32_t S = S_PIPE, LE = S_PIPE, NE = 2 * S_PIPE, RW = L::RW, EWW = PACKED ? 1 : 2;
    using RC = RowCopy<L>;
    constexpr uint32_t NONE = 0xffffffffu;
    const uint32_t lane = threadIdx.x & 31;
    const uint32_t swz = RC::sw(lane);
    if (e >= ehi) return;
    const uint32_t nch = (ehi - e + 31) >> 5;
    uint32_t* const mt = vs + S * 32 * RW;   // [S][3][32]: destination, weight, window row
    uint32_t* const er = mt + 3 * S * 32;    // [NE][32][EWW]: edge words
    uint32_t* const kr = er + NE * 32 * EWW; // [NE][32]: their window rows
    auto fetch = [&](uint32_t c) {
        const uint32_t slot = c % NE;
        const uint32_t cs = e + c * 32, t = cs + lane;
        const uint32_t below = __popc(__ballot_sync(FULL, off <= cs));
        const uint32_t rel = off - cs;
        const uint32_t starts = __reduce_or_sync(FULL, (rel - 1u < 31u) ? (1u << rel) : 0u);
        const uint32_t kk = below - 1u + __popc(starts & ((2u << lane) - 1u));
        const uint32_t mk = __shfl_sync(FULL, mask, kk);
        const uint32_t a = __shfl_sync(FULL, base, kk) + t;
        const bool ok = t < ehi && mk != 0u;
        if (ok) {
            if constexpr (PACKED)
                asm volatile("cp.async.ca.shared.global [%0], [%1], 4;" ::"r"(smem_u32(er + slot * 32 + lane)),
                             "l"(g.adj + a) : "memory");
            else
                asm volatile("cp.async.ca.shared.global [%0], [%1], 8;" ::"r"(smem_u32(er + (slot * 32 + lane) * 2)),
                             "l"(g.adjw + a) : "memory");
        }
        kr[slot * 32 + lane] = ok ? kk : NONE;
    };
    auto request = [&](uint32_t c) {  // chunk c's edge word has landed (lane-private)
        const uint32_t es = c % NE, rs = c % S;
        const uint32_t kk = kr[es * 32 + lane];
        mt[(3 * rs + 2) * 32 + lane] = kk;
        uint32_t dd = NONE;
        if (kk != NONE) {
            EdgeWord<PACKED> wd;
            if constexpr (PACKED) wd.x = er[es * 32 + lane];
            else wd.x = *reinterpret_cast<const uint2*>(er + (es * 32 + lane) * 2);
            uint32_t d, w;
            wd.decode(P.dbits, P.dmask, d, w);
            mt[(3 * rs + 0) * 32 + lane] = d;
            mt[(3 * rs + 1) * 32 + lane] = w;
            dd = d;
        }
        if constexpr (RC::C > 1) {
            constexpr uint32_t RPI = 32 / RC::C;
            const uint32_t p = lane % RC::C;
#pragma unroll
            for (uint32_t i = 0; i < RC::C; ++i) {
                const uint32_t r = i * RPI + lane / RC::C;
                const uint32_t dr = __shfl_sync(FULL, dd, r);
                if (dr != NONE)
                    RC::copy(vs + (rs * 32 + r) * RW + RC::CW4 * (p ^ RC::sw(r)), P.V + (size_t)dr * RW + RC::CW4 * p,
                             fresh);
            }
        } else if (dd != NONE) {
            RC::copy(vs + (rs * 32 + lane) * RW, P.V + (size_t)dd * RW, fresh);
        }
    };
    for (uint32_t c = 0; c < S - 1 + LE && c < nch; ++c) fetch(c);
    cp_async_commit();
    cp_async_wait<0>();
    for (uint32_t c = 0; c < S - 1; ++c) {
        if (c < nch) request(c);
        cp_async_commit();
    }
    for (uint32_t cc = 0; cc < nch; ++cc) {
        if constexpr (RC::C > 1) __syncwarp();  // every lane is done with row slot (cc - 1) % S
        if (cc + S - 1 < nch) request(cc + S - 1);
        if (cc + S - 1 + LE < nch) fetch(cc + S - 1 + LE);
        cp_async_commit();
        cp_async_wait<S - 1>();                 // chunk cc's rows (and chunk cc + S's edge words) landed
        if constexpr (RC::C > 1) __syncwarp();
        const uint32_t sr = cc % S;
        const uint32_t kk = mt[(3 * sr + 2) * 32 + lane];
        const uint32_t mk = __shfl_sync(FULL, mask, kk & 31u);
        if (kk == NONE) continue;
        ++n_read;
        const uint32_t d = mt[(3 * sr + 0) * 32 + lane];
        const typename L::Arg w = L::arg(mt[(3 * sr + 1) * 32 + lane]);
        const uint32_t* rv = vs + (sr * 32 + lane) * RW;
        const uint32_t* ru = xs + kk * RW;
        uint32_t* pv = P.V + (size_t)d * RW;
        uint32_t changed = 0;
#pragma unroll
        for (int gi = 0; gi < (int)RW / L::G; ++gi) {
            const uint32_t act = group_mask<L>(mk, gi);
            if (!act) continue;
            uint32_t uu[L::G], cc2[L::G];
#pragma unroll
            for (int j = 0; j < L::G; ++j) {
                const uint32_t i = (uint32_t)(gi * L::G + j);
                uu[j] = ru[i];
                cc2[j] = rv[((i / RC::CW4) ^ swz) * RC::CW4 + i % RC::CW4];
            }
            changed |= L::relax(pv + gi * L::G, uu, cc2, w, act, n_edges, n_upd, P.err) << (gi * L::G * L::QPW);
        }
        if (changed) {
            red_or(P.M + d, changed);
            if (set_bits) red_or(P.bitmap + (d >> 5), 1u << (d & 31));
        }
    }
    cp_async_wait<0>();
}

template <class L>  // 128 B rows (RW = 32): one window buffer, so 16 warps' buffers fit in shared memory
constexpr bool xs_double() { return L::RW <= 16; }

// ------------------------------------------------------------------ phase-1 pull (dense iterations)
// A dense phase-1 iteration as a pull over CG^R (Process, Alg 3 l.21-34, applied from the
// destination's side): every in-edge (u -> v, w) of the Core Graph is relaxed; the window's 32 rows
// are DESTINATIONS, held in xs as their current values, and a lane gathers the SOURCE row u (the
// push pipeline's fetch / request, unchanged) and forms the candidates of all Q queries.  Lanes of
// a chunk that share a destination are combined by a segmented warp scan (the kind's select, Table
// 6); the last lane of each segment compares with the xs row and, where better, updates it and
// applies the EdgeFunction ONCE for the row (vector red.min / red.max; red.or for REACH's bits) —
// one atomic per (row, chunk) instead of one per (edge, query).  Every CG in-edge is read, active or
// not: an inactive u's candidate was already applied to v (reading N6), so the extra candidates
// change nothing.  v becomes active (M) for the improved queries.
template <int KIND, bool PACKED, class L>
__device__ __forceinline__ void window_pull(const BParams& P, const GraphView& g, uint32_t* xs, uint32_t* vs,
                                            uint32_t off, uint32_t base, uint32_t vtx, uint32_t e, uint32_t ehi,
                                            uint32_t& n_edges, uint32_t& n_upd, uint32_t& n_read) {
    constexpr int EA = (L::QPW == 2 && E_AHEAD == S_PIPE) ? 2 * S_PIPE : E_AHEAD;
    constexpr int S = S_PIPE, RW = L::RW;
    constexpr uint32_t WM = L::QPW == 32 ? 0xffffffffu : (1u << L::QPW) - 1u;
    using RC = RowCopy<L>;
    constexpr uint32_t NONE = 0xffffffffu;
    const uint32_t lane = threadIdx.x & 31;
    const uint32_t swz = RC::sw(lane);
    if (e >= ehi) return;
    const uint32_t nch = (ehi - e + 31) >> 5;
    EdgeWord<PACKED> ew[EA];
    uint32_t ek[EA];
    uint32_t sw[S], sk[S];
    auto fetch = [&](uint32_t c, EdgeWord<PACKED>& wd, uint32_t& kout) {
        const uint32_t cs = e + c * 32, t = cs + lane;
        const uint32_t below = __popc(__ballot_sync(FULL, off <= cs));
        const uint32_t rel = off - cs;
        const uint32_t starts = __reduce_or_sync(FULL, (rel - 1u < 31u) ? (1u << rel) : 0u);
        const uint32_t kk = below - 1u + __popc(starts & ((2u << lane) - 1u));
        const uint32_t a = __shfl_sync(FULL, base, kk) + t;
        const bool ok = t < ehi;
        if (ok) wd.load(g, a);
        kout = ok ? kk : NONE;
    };
    auto request = [&](int slot, const EdgeWord<PACKED>& wd, uint32_t kk) {
        sk[slot] = kk;
        uint32_t dd = NONE;
        if (kk != NONE) {
            uint32_t d, w;
            wd.decode(P.dbits, P.dmask, d, w);  // d = the source u of the in-edge
            sw[slot] = w;
            dd = d;
        }
        if constexpr (RC::C > 1) {
            constexpr uint32_t RPI = 32 / RC::C;
            const uint32_t p = lane % RC::C;
#pragma unroll
            for (uint32_t i = 0; i < RC::C; ++i) {
                const uint32_t r = i * RPI + lane / RC::C;
                const uint32_t dr = __shfl_sync(FULL, dd, r);
                if (dr != NONE)
                    RC::copy(vs + (slot * 32 + r) * RW + RC::CW4 * (p ^ RC::sw(r)), P.V + (size_t)dr * RW + RC::CW4 * p,
                             false);
            }
        } else if (dd != NONE) {
            RC::copy(vs + (slot * 32 + lane) * RW, P.V + (size_t)dd * RW, false);
        }
        cp_async_commit();
    };
#pragma unroll
    for (int s = 0; s < EA; ++s) {
        ek[s] = NONE;
        if ((uint32_t)s < nch) fetch(s, ew[s], ek[s]);
    }
#pragma unroll
    for (int s = 0; s < S - 1; ++s) {
        request(s, ew[s], ek[s]);
        ek[s] = NONE;
        if ((uint32_t)(s + EA) < nch) fetch(s + EA, ew[s], ek[s]);
    }
    for (uint32_t c0 = 0; c0 < nch; c0 += EA) {
#pragma unroll
        for (int s = 0; s < EA; ++s) {
            const uint32_t cc = c0 + s;
            if (cc >= nch) break;
            const int je = (s + S - 1) % EA;
            const int jr = (s + S - 1) % S;
            if constexpr (RC::C > 1) __syncwarp();
            request(jr, ew[je], ek[je]);
            ek[je] = NONE;
            if (cc + S - 1 + EA < nch) fetch(cc + S - 1 + EA, ew[je], ek[je]);
            cp_async_wait<S - 1>();
            if constexpr (RC::C > 1) __syncwarp();
            const int sr = s % S;
            const uint32_t kk = sk[sr];
            // the candidates of this lane's in-edge for every query
            uint32_t x[RW];
            {
                const typename L::Arg w = L::arg(sw[sr]);
                const uint32_t* rv = vs + (sr * 32 + lane) * RW;
#pragma unroll
                for (int i = 0; i < RW; ++i)
                    x[i] = kk != NONE ? L::cand(rv[((i / RC::CW4) ^ swz) * RC::CW4 + i % RC::CW4], w) : 0u;
            }
            if (kk != NONE) ++n_read;
            // segmented scan (the kind's select) over the lanes of each destination row
#pragma unroll
            for (uint32_t dl = 1; dl < 32; dl <<= 1) {
                const uint32_t kd = __shfl_up_sync(FULL, kk, dl);
                const bool take = lane >= dl && kd == kk;
#pragma unroll
                for (int i = 0; i < RW; ++i) {
                    const uint32_t y = __shfl_up_sync(FULL, x[i], dl);
                    if (take) x[i] = L::sel(x[i], y);
                }
            }
            const uint32_t knext = __shfl_down_sync(FULL, kk, 1);
            const uint32_t vk = __shfl_sync(FULL, vtx, kk & 31u);
            const bool leader = kk != NONE && (lane == 31 || knext != kk);
            if (leader) {
                uint32_t* row = xs + kk * RW;
                uint32_t* pv = P.V + (size_t)vk * RW;
                uint32_t imp = 0, over = 0;
#pragma unroll
                for (int i = 0; i < RW; ++i) {
                    const uint32_t c = row[i];
                    const uint32_t im = L::improve(x[i], c) & WM;
                    imp |= im << (i * L::QPW);
                    if constexpr (L::QPW == 2) over |= (uint32_t)L::overflow(x[i], c);
                    if (im) row[i] = L::sel(x[i], c);
                }
                if (over) atomicOr(P.err, ERR_LANE_OVERFLOW);
                if (imp) {  // the row's EdgeFunction, once
                    if constexpr (L::QPW == 2) {
#pragma unroll
                        for (int h = 0; h < RW / 4; ++h) {
                            if (!((imp >> (8 * h)) & 0xffu)) continue;
                            if constexpr (KIND == CG_SSWP)
                                asm volatile("red.relaxed.gpu.global.max.noftz.v4.f16x2 [%0], {%1,%2,%3,%4};" ::"l"(pv + 4 * h),
                                             "r"(x[4 * h]), "r"(x[4 * h + 1]), "r"(x[4 * h + 2]), "r"(x[4 * h + 3]) : "memory");
                            else
                                asm volatile("red.relaxed.gpu.global.min.noftz.v4.f16x2 [%0], {%1,%2,%3,%4};" ::"l"(pv + 4 * h),
                                             "r"(x[4 * h]), "r"(x[4 * h + 1]), "r"(x[4 * h + 2]), "r"(x[4 * h + 3]) : "memory");
                        }
                    } else {
#pragma unroll
                        for (int i = 0; i < RW; ++i) {
                            if (!((imp >> (i * L::QPW)) & WM)) continue;
                            if constexpr (L::QPW == 32) red_or(pv + i, x[i]);
                            else Op<KIND>::edge_fn(pv + i, x[i]);
                        }
                    }
                    red_or(P.M + vk, imp);
                    n_upd += __popc(imp);
                    n_edges += __popc(imp);
                }
            }
            __syncwarp();  // the leaders' xs updates are seen by the next chunk
        }
    }
    cp_async_wait<0>();
}

// The whole in-edge list of CG^R (static: vertices with CG in-edges, vertex order) split evenly over
// all warps; windows of 32 destinations as in relax_range.
template <int KIND, bool PACKED, class L>
__device__ void relax_pull_all(const BParams& P, uint32_t* xs, uint32_t* vs, uint32_t& n_edges, uint32_t& n_upd,
                               uint32_t& n_read) {
    constexpr int RW = L::RW;
    using RC = RowCopy<L>;
    const GraphView& g = P.RC;
    const uint32_t count = P.pl_count, E = P.pl_E;
    const uint32_t lane = threadIdx.x & 31;
    const uint32_t gw = blockIdx.x * BW + (threadIdx.x >> 5);
    const uint64_t NW = (uint64_t)gridDim.x * BW;
    const uint32_t e0 = (uint32_t)((uint64_t)E * gw / NW), e1 = (uint32_t)((uint64_t)E * (gw + 1) / NW);
    if (e0 >= e1) return;
    uint32_t lo = 0, hi = count;  // 32-ary search: the window holding edge e0
    while (hi - lo > 32) {
        const uint32_t step = (hi - lo + 31) / 32;
        const uint32_t p = lo + lane * step;
        const bool le = p < hi && __ldg(P.pl_lo + p) <= e0;
        const uint32_t k = 31 - __clz(__ballot_sync(FULL, le));
        const uint32_t nlo = lo + k * step;
        hi = min(hi, nlo + step);
        lo = nlo;
    }
    {
        const uint32_t p = lo + lane;
        const bool le = p < hi && __ldg(P.pl_lo + p) <= e0;
        lo += 31 - __clz(__ballot_sync(FULL, le));
    }
    auto list_load = [&](uint32_t i0, uint32_t& v, uint32_t& off) {
        const uint32_t idx = i0 + lane;
        v = 0;
        off = E;
        if (idx < count) {
            v = __ldg(P.pl_v + idx);
            off = __ldg(P.pl_lo + idx);
        }
    };
    auto rows_async = [&](uint32_t* buf, uint32_t v, uint32_t i0) {  // the window's destination rows -> buf
#pragma unroll
        for (uint32_t r = 0; r < RC::C; ++r) {
            const uint32_t f = r * 32 + lane, row = f / RC::C, c = f % RC::C;
            const uint32_t vr = __shfl_sync(FULL, v, row);
            if (i0 + row < count) RC::copy(buf + row * RW + c * RC::CW4, P.V + (size_t)vr * RW + c * RC::CW4, true);
        }
        cp_async_commit();
    };
    constexpr bool DB = xs_double<L>();  // the next window's rows are copied while this one runs
    uint32_t i = lo, e = e0, cv, coff, nv, noff;
    list_load(i, cv, coff);
    rows_async(xs, cv, i);
    list_load(i + 32, nv, noff);
    uint32_t buf = 0;
    for (;;) {
        const uint32_t wend = (i + 32 < count) ? __shfl_sync(FULL, noff, 0) : E;
        const uint32_t ehi = min(e1, wend);
        const bool more = ehi < e1;
        uint32_t mv = 0, moff = E;
        if (more) {
            if constexpr (DB) rows_async(xs + (buf ^ 1) * 32 * RW, nv, i + 32);
            list_load(i + 64, mv, moff);
        }
        if (DB && more) cp_async_wait<1>();
        else cp_async_wait<0>();
        __syncwarp();
        window_pull<KIND, PACKED, L>(P, g, xs + buf * 32 * RW, vs, coff, 0u, cv, e, ehi, n_edges, n_upd, n_read);
        __syncwarp();
        if (!more) break;
        if constexpr (!DB) rows_async(xs, nv, i + 32);
        e = ehi;
        i += 32;
        if constexpr (DB) buf ^= 1;
        cv = nv;
        coff = noff;
        nv = mv;
        noff = moff;
    }
}

// The window's 32 rows (all Q queries) into shared memory, coalesced (RW words per row)
template <class L>
__device__ __forceinline__ void load_rows(const BParams& P, uint32_t* xs, uint32_t v, uint32_t i, uint32_t count) {
    const uint32_t lane = threadIdx.x & 31;
    __syncwarp();
#pragma unroll
    for (int r = 0; r < L::RW; ++r) {
        const uint32_t f = r * 32 + lane;  // flat index row*RW + word
        const uint32_t vr = __shfl_sync(FULL, v, f / L::RW);
        xs[f] = (i + f / L::RW < count) ? ld_cg(P.V + (size_t)vr * L::RW + f % L::RW) : 0u;
    }
    __syncwarp();
}

// first list entry of the warp's edge range: 32-ary search over the list's edge offsets
__device__ __forceinline__ uint32_t first_entry(const BParams& P, uint32_t count, uint32_t e0) {
    const uint32_t lane = threadIdx.x & 31;
    uint32_t lo = 0, hi = count;
    while (hi - lo > 32) {
        const uint32_t step = (hi - lo + 31) / 32;
        const uint32_t p = lo + lane * step;
        const bool le = p < hi && ld_cg(P.lo + p) <= e0;
        const uint32_t k = 31 - __clz(__ballot_sync(FULL, le));
        const uint32_t nlo = lo + k * step;
        hi = min(hi, nlo + step);
        lo = nlo;
    }
    const uint32_t p = lo + lane;
    const bool le = p < hi && ld_cg(P.lo + p) <= e0;
    return lo + 31 - __clz(__ballot_sync(FULL, le));
}

// S2 over the compacted list: the iteration's E list edges split evenly over all warps; a warp
// slides 32-entry windows (a hub row is shared by as many warps and CTAs as needed).  Windows
// are prefetched one ahead: while window i's edges run, window i+1's source rows are already
// being copied (cp.async) into the other half of xs and window i+2's list entries are loading.
template <int KIND, bool PACKED, class L>
__device__ void relax_range(const BParams& P, const GraphView& g, uint32_t count, uint32_t E, uint32_t e0, uint32_t e1,
                            uint32_t* xs, uint32_t* vs, bool set_bits, bool fresh, uint32_t& n_edges, uint32_t& n_upd,
                            uint32_t& n_read) {
    constexpr int RW = L::RW;
    using RC = RowCopy<L>;
    const uint32_t lane = threadIdx.x & 31;
    if (e0 >= e1) return;
    auto list_load = [&](uint32_t i0, uint32_t& v, uint32_t& off, uint32_t& mask) {
        const uint32_t idx = i0 + lane;
        v = 0;
        off = E;
        mask = 0;
        if (idx < count) {
            v = ld_cg(P.lv + idx);
            off = ld_cg(P.lo + idx);
            mask = ld_cg(P.lm + idx);
        }
    };
    auto rows_async = [&](uint32_t* buf, uint32_t v, uint32_t i0) {  // the window's 32 rows -> buf
#pragma unroll
        for (uint32_t r = 0; r < RC::C; ++r) {
            const uint32_t f = r * 32 + lane, row = f / RC::C, c = f % RC::C;
            const uint32_t vr = __shfl_sync(FULL, v, row);
            if (i0 + row < count) RC::copy(buf + row * RW + c * RC::CW4, P.V + (size_t)vr * RW + c * RC::CW4, false);
        }
        cp_async_commit();
    };
    constexpr bool DB = xs_double<L>();  // next window's rows copied while this one runs
    uint32_t i = first_entry(P, count, e0), e = e0;
    uint32_t cv, coff, cmask, nv, noff, nmask;
    list_load(i, cv, coff, cmask);
    uint32_t cbase = i + lane < count ? __ldg(g.ptr + cv) - coff : 0u;
    rows_async(xs, cv, i);
    list_load(i + 32, nv, noff, nmask);
    uint32_t buf = 0;
    for (;;) {
        const uint32_t wend = (i + 32 < count) ? __shfl_sync(FULL, noff, 0) : E;  // lo[i + 32]
        const uint32_t ehi = min(e1, wend);
        const bool more = ehi < e1;
        uint32_t nbase = 0, mv = 0, moff = E, mmask = 0;
        if (more) {
            nbase = i + 32 + lane < count ? __ldg(g.ptr + nv) - noff : 0u;
            if constexpr (DB) rows_async(xs + (buf ^ 1) * 32 * RW, nv, i + 32);
            list_load(i + 64, mv, moff, mmask);
        }
        if (DB && more) cp_async_wait<1>();  // this window's rows (the next window's may still fly)
        else cp_async_wait<0>();
        __syncwarp();
        if constexpr (edge_smem<L>())
            window_edges_sm<KIND, PACKED, L>(P, g, xs + buf * 32 * RW, vs, coff, cbase, cmask, e, ehi, set_bits, fresh,
                                             n_edges, n_upd, n_read);
        else
            window_edges<KIND, PACKED, L>(P, g, xs + buf * 32 * RW, vs, coff, cbase, cmask, e, ehi, set_bits, fresh,
                                          n_edges, n_upd, n_read);
        __syncwarp();  // every lane is done with this window's rows before they are overwritten
        if (!more) break;
        if constexpr (!DB) rows_async(xs, nv, i + 32);
        e = ehi;
        i += 32;
        if constexpr (DB) buf ^= 1;
        cv = nv;
        coff = noff;
        cmask = nmask;
        cbase = nbase;
        nv = mv;
        noff = moff;
        nmask = mmask;
    }
}

// The iteration's E list edges over all warps: a static half split evenly (edge-balanced), then
// — for iterations long enough to amortise a tile's list search — the rest in tiles taken from
// a per-iteration counter, so warps slowed by contended EdgeFunctions (phase 1's hub rows) do
// not hold the grid barrier (trace: the last CTA finished 33 % after the first without it).
#ifndef CGB_DYN_MIN
#define CGB_DYN_MIN 1024u  // edges per warp below which the split stays fully static (measured 512 / 1024 / 2048)
#endif
template <int KIND, bool PACKED, class L>
__device__ void relax_b(const BParams& P, const GraphView& g, uint32_t count, uint32_t E, uint32_t* xs, uint32_t* vs,
                        bool set_bits, bool fresh, uint32_t& n_edges, uint32_t& n_upd, uint32_t& n_read,
                        unsigned long long* tiles) {
    const uint32_t lane = threadIdx.x & 31;
    const uint32_t gw = blockIdx.x * BW + (threadIdx.x >> 5);
    const uint64_t NW = (uint64_t)gridDim.x * BW;
    const bool dyn = tiles != nullptr && (uint64_t)E >= NW * CGB_DYN_MIN;
#ifndef CGB_DYN_STATIC
#define CGB_DYN_STATIC 2  // 1 / (static share of a dynamic iteration's edges)
#endif
#ifndef CGB_DYN_TPW
#define CGB_DYN_TPW 4     // dynamic tiles per warp (measured on C2: 1 -> 11.79 K q/s, 2 -> 11.86 K (static 1/4), 4 -> 12.24 K)
#endif
    const uint32_t Es = dyn ? E / CGB_DYN_STATIC : E;
    const uint32_t T = dyn ? max(1024u / CGB_DYN_TPW, (uint32_t)((E - Es + NW * CGB_DYN_TPW - 1) / (NW * CGB_DYN_TPW))) : 0u;
    uint32_t a = (uint32_t)((uint64_t)Es * gw / NW), b = (uint32_t)((uint64_t)Es * (gw + 1) / NW);
    for (;;) {  // one call site: the range body is inlined once
        relax_range<KIND, PACKED, L>(P, g, count, E, a, b, xs, vs, set_bits, fresh, n_edges, n_upd, n_read);
        if (!dyn) break;
        unsigned long long t = 0;
        if (lane == 0) t = atomicAdd(tiles, 1ull);
        t = __shfl_sync(FULL, t, 0);
        const uint64_t a64 = Es + t * T;
        if (a64 >= E) break;
        a = (uint32_t)a64;
        b = (uint32_t)(a64 + T < E ? a64 + T : E);
    }
}

// ------------------------------------------------------------------ NEXT-1 pull (Reduced(E))
// The list holds vertices v with uncertified queries (mask) and their IN-edge offsets; a lane
// takes an in-edge (u -> v, w) of the edge-balanced split and, for each uncertified query q,
// applies the Table 6 Needed / EdgeFunction to Val(v): all pushes INTO uncertified vertices in
// one sweep, none into certified ones (their in-edges are removed).
template <int KIND, bool PACKED, class L>
__device__ void relax_pull(const BParams& P, uint32_t count, uint32_t E, uint32_t* xs, uint32_t& n_edges,
                           uint32_t& n_upd, uint32_t& n_read) {
    constexpr int U = 2, RW = L::RW;
    const GraphView& g = P.R;
    const uint32_t lane = threadIdx.x & 31;
    const uint32_t gw = blockIdx.x * BW + (threadIdx.x >> 5);
    const uint64_t NW = (uint64_t)gridDim.x * BW;
    const uint32_t e0 = (uint32_t)((uint64_t)E * gw / NW), e1 = (uint32_t)((uint64_t)E * (gw + 1) / NW);
    if (e0 >= e1) return;
    uint32_t i = first_entry(P, count, e0), e = e0;
    for (;;) {
        const uint32_t idx = i + lane;
        uint32_t off = E, base = 0, v = 0, mask = 0;
        if (idx < count) {
            v = ld_cg(P.lv + idx);
            off = ld_cg(P.lo + idx);
            mask = ld_cg(P.lm + idx);
            base = __ldg(g.ptr + v) - off;
        }
        load_rows<L>(P, xs, v, i, count);  // current rows of the pulling vertices (Needed test)
        const uint32_t wend = (i + 32 < count) ? ld_cg(P.lo + i + 32) : E;
        const uint32_t ehi = min(e1, wend);
        for (; e < ehi; e += 32 * U) {
            uint32_t k[U], mk[U], vk[U];
            bool ok[U];
            EdgeWord<PACKED> wd[U];
#pragma unroll
            for (int u = 0; u < U; ++u) {
                const uint32_t t = e + u * 32 + lane;
                uint32_t kk = 0;
#pragma unroll
                for (uint32_t st = 16; st > 0; st >>= 1)
                    if (__shfl_sync(FULL, off, kk + st) <= t) kk += st;
                k[u] = kk;
                mk[u] = __shfl_sync(FULL, mask, kk);
                vk[u] = __shfl_sync(FULL, v, kk);
                const uint32_t a = __shfl_sync(FULL, base, kk) + t;
                ok[u] = t < ehi && mk[u] != 0u;
                if (ok[u]) wd[u].load(g, a);
            }
#pragma unroll
            for (int u = 0; u < U; ++u) {
                if (!ok[u]) continue;
                uint32_t src, w0;
                wd[u].decode(P.dbits, P.dmask, src, w0);
                const typename L::Arg w = L::arg(w0);
                ++n_read;
                const uint32_t* ru = P.V + (size_t)src * RW;  // u's row (L1: a stale value is never better)
                uint32_t* pv = P.V + (size_t)vk[u] * RW;
                uint32_t changed = 0;
#pragma unroll
                for (int gi = 0; gi < RW / L::G; ++gi) {
                    const uint32_t act = group_mask<L>(mk[u], gi);
                    if (!act) continue;
                    uint32_t uu[L::G], cc2[L::G];
#pragma unroll
                    for (int j = 0; j < L::G; ++j) {
                        uu[j] = ld_l1(ru + gi * L::G + j);
                        cc2[j] = xs[k[u] * RW + gi * L::G + j];
                    }
                    changed |= L::relax(pv + gi * L::G, uu, cc2, w, act, n_edges, n_upd, P.err) << (gi * L::G * L::QPW);
                }
                if (changed) red_or(P.M + vk[u], changed);  // v pushes onward for those queries
            }
        }
        if (ehi >= e1) break;
        e = ehi;
        i += 32;
    }
}

// Batch-total count c (per thread) split evenly over the nq queries' counter k: block sum,
// then thread 0 adds total/nq to each (the remainder to the first).
__device__ __forceinline__ void block_add_split(unsigned long long* stats, int q0, int nq, int k, unsigned long long c,
                                                unsigned long long* sm) {
    const unsigned long long t = block_sum<BW, unsigned long long>(c, sm);
    if (threadIdx.x == 0 && t)
        for (int b = 0; b < nq; ++b)
            atomicAdd(stats + (size_t)(q0 + b) * NSTAT + k, t / nq + (b == 0 ? t % nq : 0));
}

// Add a per-thread count to query (tid % Q)'s counter k (the thread's query is fixed in loops
// whose stride is a multiple of Q).
template <int Q>
__device__ __forceinline__ void per_query_add(unsigned long long* stats, int q0, int nq, int k, unsigned long long c) {
#pragma unroll
    for (int o = Q; o < 32; o <<= 1) c += __shfl_xor_sync(FULL, c, o);
    const uint32_t lane = threadIdx.x & 31;
    if (lane < (uint32_t)Q && (int)lane < nq && c) atomicAdd(stats + (size_t)(q0 + lane) * NSTAT + k, c);
}

// value of query q at v, caller encoding
template <class L>
__device__ __forceinline__ uint32_t value_of(const uint32_t* V, uint32_t v, uint32_t q) {
    return L::decode(ld_cg(V + (size_t)v * L::RW + q / L::QPW), q % L::QPW);
}

#ifndef CGB_TSTORE
#define CGB_TSTORE 0
#endif
__device__ __forceinline__ void tstore(uint32_t* p, uint32_t x) {
    if (CGB_TSTORE == 0) __stcs(p, x);
    else if (CGB_TSTORE == 1) *p = x;
    else __stcg(p, x);
}

// rows -> dst[(q0+q)*n + v] for q < nq, 32 vertices (a tile) per warp through shared memory:
// each lane decodes its vertex's Q values and every query's 32 values leave as one 128 B
// streaming store.  16 B-row layouts stage tiles two ahead in the warp's (then idle) S2 row
// ring `vs` with cp.async, so the row reads of later tiles overlap this tile's stores; the
// staged tile is copied into the padded tile in xs (conflict-free column reads).
template <class L>
__device__ void transpose_out(const BParams& P, uint32_t* dst, int q0, int nq, uint32_t* xs, uint32_t* vs) {
    constexpr int RW = L::RW;
    const uint32_t lane = threadIdx.x & 31;
    const uint32_t gw = blockIdx.x * BW + (threadIdx.x >> 5);
    const uint32_t NW = gridDim.x * BW;
    const uint32_t T = (P.n + 31) / 32;  // tiles
    if constexpr (RW % 4 == 0) {
        constexpr int NC = RW / 4;          // 16 B pieces per lane per tile
        constexpr uint32_t TW = 32 * RW;    // staged words per tile
        static_assert(2 * TW <= S_PIPE * 32 * RW, "two staged tiles fit the row ring");
        auto stage = [&](uint32_t tile, int slot) {
            if (tile < T) {
#pragma unroll
                for (int r = 0; r < NC; ++r) {
                    const uint32_t f = r * 32 + lane, row = f / NC, c = f % NC;
                    const uint32_t v = tile * 32 + row;
                    if (v < P.n) cp_async16_cg(vs + slot * TW + row * RW + 4 * c, P.V + (size_t)v * RW + 4 * c);
                }
            }
            cp_async_commit();
        };
        stage(gw, 0);
        stage(gw + NW, 1);
        int slot = 0;
        for (uint32_t tile = gw; tile < T; tile += NW) {
            cp_async_wait<1>();
            __syncwarp();
#pragma unroll
            for (int r = 0; r < NC; ++r) {
                const uint32_t f = r * 32 + lane, row = f / NC, c = f % NC;
                const uint4 x = *reinterpret_cast<const uint4*>(vs + slot * TW + row * RW + 4 * c);
                uint32_t* d = xs + row * (RW + 1) + 4 * c;
                d[0] = x.x;
                d[1] = x.y;
                d[2] = x.z;
                d[3] = x.w;
            }
            __syncwarp();
            stage(tile + 2 * NW, slot);  // refill the slot just read
            const uint32_t v = tile * 32 + lane;
            if (v < P.n)
                for (int q = 0; q < nq; ++q)
                    tstore(dst + (size_t)(q0 + q) * P.n + v, L::decode(xs[lane * (RW + 1) + q / L::QPW], q % L::QPW));
            __syncwarp();  // xs is rewritten by the next tile
            slot ^= 1;
        }
        cp_async_wait<0>();
    } else {
        for (uint32_t tile = gw; tile < T; tile += NW) {
            __syncwarp();
#pragma unroll
            for (int r = 0; r < RW; ++r) {
                const uint32_t f = r * 32 + lane;
                const uint32_t v = tile * 32 + f / RW;
                xs[(f / RW) * (RW + 1) + f % RW] = v < P.n ? __ldcg(P.V + (size_t)v * RW + f % RW) : 0u;
            }
            __syncwarp();
            const uint32_t v = tile * 32 + lane;
            if (v < P.n)
                for (int q = 0; q < nq; ++q)
                    __stcs(dst + (size_t)(q0 + q) * P.n + v, L::decode(xs[lane * (RW + 1) + q / L::QPW], q % L::QPW));
        }
    }
}

// Narrow output formats (cg_out_format): the same values, fewer bytes on the wire.
//   CG_OUT_U16:  row q = n uint16 values, InitVal / SourceInitVal 0xFFFFFFFF as 0xFFFF; a value
//                >= 0xFFFF that is not 0xFFFFFFFF cannot be represented (ERR_NARROW -> CG_EOVERFLOW)
//   CG_OUT_BITS: REACH only, row q = ceil(n/32) words, bit (v % 32) of word v / 32 = Val(v)
// 32 vertices (a tile) per warp: the tile's rows through the padded shared tile (U16), or the
// 32 x 32 bit matrix of a REACH tile transposed with one ballot per query (BITS).
template <class L>
constexpr uint32_t vs_words();
template <class L>
__device__ void transpose_narrow(const BParams& P, int q0, int nq, uint32_t* xs, uint32_t* buf) {
    constexpr int RW = L::RW;
    const uint32_t lane = threadIdx.x & 31;
    const uint32_t gw = blockIdx.x * BW + (threadIdx.x >> 5);
    const uint32_t NW = gridDim.x * BW;
    const uint32_t T = (P.n + 31) / 32;  // tiles
    if constexpr (L::QPW == 32) {  // bit lanes: CG_OUT_BITS (the host admits REACH only)
      if (P.out_fmt == CG_OUT_BITS) {
        uint32_t* dst = static_cast<uint32_t*>(P.out);
        for (uint32_t tile = gw; tile < T; tile += NW) {
            const uint32_t v = tile * 32 + lane;
            const uint32_t row = v < P.n ? ld_cg(P.V + v) : 0u;
            uint32_t mine = 0;
            for (int q = 0; q < nq; ++q) {
                const uint32_t b = __ballot_sync(FULL, (row >> q) & 1u);
                if ((int)lane == q) mine = b;
            }
            if ((int)lane < nq) __stcs(dst + (size_t)(q0 + lane) * T + tile, mine);
        }
        return;
      }
    }
    if (P.out_fmt != CG_OUT_U16) return;
    static_assert(65 * (L::RW + 1) <= vs_words<L>(), "the u16 tile fits the warp's row ring");
    uint16_t* dst = static_cast<uint16_t*>(P.out);
    bool over = false;
    // 64 vertices per warp tile, every row written with 4 B stores of vertex PAIRS (128 B per warp
    // instruction): a pair must start at an even u16 index of the output, so a row whose start
    // (q0 + q) * n is odd pairs (t0 - 1, t0), (t0 + 1, t0 + 2), ...: the tile's buffer holds the 65
    // value rows of vertices t0 - 1 .. t0 + 63 (row stride RW + 1 words), and one more tile than
    // n / 64 covers the last vertex of the odd rows.  Unpaired ends use a 2 B store.
    constexpr uint32_t RP = RW + 1;
    const uint32_t T2 = P.n / 64 + 1;
    auto val16 = [&](uint32_t r, int q) -> uint32_t {
        const uint32_t x = L::decode(buf[r * RP + q / L::QPW], q % L::QPW);
        over |= x >= 0xffffu && x != 0xffffffffu;
        return x >= 0xffffu ? 0xffffu : x;
    };
    for (uint32_t tile = gw; tile < T2; tile += NW) {
        const uint32_t t0 = tile * 64;
        __syncwarp();
#pragma unroll
        for (uint32_t f = lane; f < 65u * RW; f += 32) {  // buffer row r = vertex t0 - 1 + r
            const uint32_t r = f / RW, wd = f % RW, v = t0 - 1u + r;  // (t0 = 0, r = 0: v wraps past n)
            buf[r * RP + wd] = v < P.n ? __ldcg(P.V + (size_t)v * RW + wd) : 0u;
        }
        __syncwarp();
        for (int q = 0; q < nq; ++q) {
            const uint64_t base = (uint64_t)(q0 + q) * P.n;
            const uint32_t par = (uint32_t)(base & 1u);
            const uint32_t va = t0 + 2 * lane - par;  // the lane's pair: vertices va, va + 1
            const uint32_t ra = 2 * lane + 1 - par;   // their buffer rows ra, ra + 1
            const bool oka = va < P.n, okb = va + 1u < P.n;  // (va = -1 wraps past n)
            const uint32_t lo = val16(ra, q), hi = val16(ra + 1, q);
            if (oka && okb) __stcs(reinterpret_cast<unsigned int*>(dst + base + va), lo | (hi << 16));
            else if (oka) __stcs(reinterpret_cast<unsigned short*>(dst + base + va), (unsigned short)lo);
            else if (okb) __stcs(reinterpret_cast<unsigned short*>(dst + base + (uint32_t)(va + 1u)), (unsigned short)hi);
        }
    }
    if (over) atomicOr(P.err, ERR_NARROW);
}

template <class L>  // per warp, 16 B aligned: one or two 32-row windows (S2) or the padded transpose tile
constexpr uint32_t xs_words() {
    return (xs_double<L>() ? 2 : 1) * 32 * L::RW > ((32 * (L::RW + 1) + 3) & ~3u) ? (xs_double<L>() ? 2 : 1) * 32 * L::RW
                                                                                 : ((32 * (L::RW + 1) + 3) & ~3u);
}
template <class L>
constexpr uint32_t vs_words() {  // row ring + metadata ring (+ edge ring and its window rows)
    return S_PIPE * 32 * L::RW + 3 * S_PIPE * 32 + (edge_smem<L>() ? 2 * S_PIPE * 32 * 3 : 0);
}

template <int KIND, bool PACKED, class L>
__global__ void __launch_bounds__(BT, BT <= 512 ? 512 / BT : 1) batch_kernel(BParams P) {
    constexpr int Q = L::Q, RW = L::RW;
    __shared__ uint32_t sm_cnt[2 * BW + 2];
    __shared__ unsigned long long sm_red[BW];
    // dynamic shared memory: per warp xs (window rows / transpose tile), then per warp the
    // S_PIPE-stage value-row ring vs, then Q*2*64 source hub values sh (certificates)
    extern __shared__ __align__(16) uint32_t dsm[];
    uint32_t* xs = dsm + (threadIdx.x >> 5) * xs_words<L>();
    uint32_t* vs = dsm + BW * xs_words<L>() + (threadIdx.x >> 5) * vs_words<L>();
    uint32_t* sh = dsm + BW * (xs_words<L>() + vs_words<L>());
    // the u32-lane re-run of a binary16 call (reading N3) runs only if that call overflowed;
    // every CTA reads the same word, so the whole grid exits together
    if (P.guard && !(ld_cg(P.guard) & ERR_LANE_OVERFLOW)) return;
    unsigned long long epoch = 0;
    const uint64_t tid = blockIdx.x * (uint64_t)BT + threadIdx.x;
    const uint64_t nthreads = (uint64_t)gridDim.x * BT;
    uint32_t ring = 0;
    // thread 0's bookkeeping lives in shared memory (not registers live across the loop):
    // sticky errors of this launch, and the pass's start / phase-switch times (stats)
    __shared__ uint32_t sm_err;
    __shared__ unsigned long long sm_t[4];  // pass start, phase switch, phase 2 start, values written
    if (threadIdx.x == 0) sm_err = 0u;
    if (threadIdx.x <= 64) s_rcp[threadIdx.x] = threadIdx.x ? __frcp_rn((float)threadIdx.x) : 0.0f;
    __syncthreads();

    // kernel-level trace marks (tid 0): [cap-1] = {entry, seeds done, loop done, exit} of batch 0
    unsigned long long* kt = (P.trace && tid == 0) ? P.trace + 5ull * (P.trace_cap - 1) : nullptr;
    if (kt) kt[0] = global_ns();
    for (int q0 = 0; q0 < P.n_src; q0 += Q) {
        const int nq = min(Q, P.n_src - q0);
        if (P.stats && tid == 0) sm_t[0] = sm_t[1] = sm_t[2] = global_ns();
        // Alg 3 l.4, l.6 for every query of the batch; masks cleared
        if constexpr (RW % 4 == 0 && !InitOf<L>::ALL_ACTIVE) {  // 16 B stores
            const uint32_t iw = L::init_word();
            const uint4 x = make_uint4(iw, iw, iw, iw);
            uint4* V4 = reinterpret_cast<uint4*>(P.V);
            for (uint64_t i = tid; i < (uint64_t)P.n * (RW / 4); i += nthreads) V4[i] = x;
        } else {
            for (uint64_t i = tid; i < (uint64_t)P.n * RW; i += nthreads) P.V[i] = InitOf<L>::at(i);
        }
        for (uint64_t v = tid; v < P.n; v += nthreads) P.M[v] = InitOf<L>::ALL_ACTIVE ? 1u : 0u;
        grid_sync(P.ctrl, epoch);
        for (int b = 0; b < nq && !InitOf<L>::ALL_ACTIVE; ++b) {
            const uint32_t s = __ldg(P.srcs + q0 + b);
            if (s >= P.n) {  // CG_EINVAL, reported through the sticky word; the row stays InitVal
                if (threadIdx.x == 0) sm_err |= ERR_SOURCE;
                continue;
            }
            uint32_t* col = P.V + b / L::QPW;
            if (tid == 0) L::seed(col + (size_t)s * RW, b % L::QPW, L::src_val());
            // l.5, l.10: out-neighbours of s in G
            const uint32_t r0 = __ldg(P.G.ptr + s), r1 = __ldg(P.G.ptr + s + 1);
            for (uint64_t e = r0 + tid; e < r1; e += nthreads) {
                EdgeWord<PACKED> wd;
                wd.load(P.G, (uint32_t)e);
                uint32_t d, w;
                wd.decode(P.dbits, P.dmask, d, w);
                L::seed(col + (size_t)d * RW, b % L::QPW, L::nb_val(w));
                red_or(P.M + d, 1u << b);
                red_or(P.bitmap + (d >> 5), 1u << (d & 31));
            }
        }
        if (P.HB) {  // the sources' hub values (certificates), per block
            for (uint32_t i = threadIdx.x; i < (uint32_t)nq * 2 * P.K; i += BT) {
                const uint32_t b = i / (2 * P.K), k = i % (2 * P.K);
                const uint32_t s = __ldg(P.srcs + q0 + b);
                const uint32_t col = k < P.K ? k : P.KP + (k - P.K);
                sh[i] = s < P.n ? __ldg(P.HB + (size_t)s * 2 * P.KP + col) : 0u;
            }
        }
        grid_sync(P.ctrl, epoch);
        if (kt && q0 == 0) kt[1] = global_ns();

        int phase = P.two_phase ? 1 : 2;
        bool predicate = false;  // this iteration's S1 seeds Active with the impacted vertices
        bool bits = !InitOf<L>::ALL_ACTIVE;  // the frontier is in the bitmap (seeds set bits), else in M
        bool pull = false;       // this iteration is the NEXT-1 pull over uncertified vertices
        uint32_t iters = 0, n_edges = 0, n_upd = 0, n_read = 0;  // (edge, query) pairs / edge reads
        for (;;) {
            // phase 2's first sweep (Alg 3 l.15 seeding, `predicate`) relaxes G minus the CG:
            // every CG edge is at its fixpoint after phase 1 (reading N7)
            const GraphView& g = (phase == 1) ? P.C : (predicate && P.Rst.ptr) ? P.Rst : P.G;
            const bool fresh = (P.fresh >> (phase - 1)) & 1u;
            const int slot = ring & 3;
            unsigned long long* ctr = P.ctrl + CT0 + CTS * slot;
            if (tid == 0) {
                unsigned long long* z = P.ctrl + CT0 + CTS * ((ring + 2) & 3);
                z[0] = z[1] = z[2] = 0ull;
            }
            const unsigned long long t_s0 = (P.trace && tid == 0) ? global_ns() : 0ull;
            const int mode = pull ? F_UNCERT : predicate ? F_IMPACTED : bits ? F_BITS : F_MASKS;
            if (mode == F_BITS) {
                compact_bits(P, g, ctr + CT_LIST, ctr + CT_ACTIVE, sm_cnt);
            } else {
                if (mode != F_MASKS) {  // impacted (l.15) / uncertified (NEXT-1) queries into M
                    mark_masks<KIND, L>(P, mode, sh, nq);
                    grid_sync(P.ctrl, epoch);
                }
                compact_masks(P, pull ? P.R : g, ctr + CT_LIST, ctr + CT_ACTIVE, sm_cnt);
            }
            grid_sync(P.ctrl, epoch);
            ++ring;
            const unsigned long long ce = ld_cg64(ctr + CT_LIST);
            const uint32_t count = (uint32_t)(ce >> 32), E = (uint32_t)ce;
            const uint32_t tr = ring - 1;
            if (P.trace && tid == 0 && tr + 1 < P.trace_cap) {
                unsigned long long* t = P.trace + 5ull * tr;
                t[0] = t_s0;
                t[1] = global_ns();
                t[2] = 0;
                t[3] = ((unsigned long long)phase << 62) | ((unsigned long long)q0 << 32) | count;
                t[4] = (ld_cg64(ctr + CT_ACTIVE) << 32) | E;
            }
            if (P.stats && tid == 0) {
                const unsigned long long a = ld_cg64(ctr + CT_ACTIVE);
                for (int b = 0; b < nq; ++b)  // union frontier, reported for every query of the batch
                    atomicAdd(P.stats + (size_t)(q0 + b) * NSTAT + (phase == 1 ? ST_F1 : ST_F2), a);
            }
            if (E == 0 && pull) {  // nothing uncertified has an in-edge: phase 2 is already final
                pull = false;
                bits = false;
            }
            if (E == 0) {
                if (P.stats) {  // batch totals, attributed evenly to the batch's queries
                    block_add_split(P.stats, q0, nq, phase == 1 ? ST_E1 : ST_E2, n_edges, sm_red);
                    block_add_split(P.stats, q0, nq, phase == 1 ? ST_U1 : ST_U2, n_upd, sm_red);
                    block_add_split(P.stats, q0, nq, phase == 1 ? ST_S1 : ST_S2, n_read, sm_red);
                    if (tid < (uint64_t)nq)
                        atomicAdd(P.stats + (size_t)(q0 + tid) * NSTAT + (phase == 1 ? ST_IT1 : ST_IT2),
                                  (unsigned long long)iters);
                }
                n_edges = n_upd = n_read = 0;
                iters = 0;
                if (phase == 1) {
                    if (P.stats && tid == 0) sm_t[1] = global_ns();  // (the counters' own passes excluded)
                    if (P.p1) transpose_out<L>(P, P.p1, q0, nq, xs, vs);
                    if (P.stats) {  // impacted per query (Alg 3 l.15); the thread's query q is fixed
                        const uint32_t q = (uint32_t)(tid % Q);
                        const uint32_t init = L::decode(L::init_word(), 0);
                        unsigned long long c = 0;
                        for (uint64_t v = tid / Q; v < P.n; v += nthreads / Q)
                            c += value_of<L>(P.V, (uint32_t)v, q) != init;
                        per_query_add<Q>(P.stats, q0, nq, ST_IMP, c);
                    }
                    // the p1 / impacted reads must finish before phase 2 updates V
                    if (P.p1 || P.stats) grid_sync(P.ctrl, epoch);
                    if (P.stats && tid == 0) sm_t[2] = global_ns();
                    phase = 2;
                    if (P.reduced) pull = true;   // Reduced(E): pull into uncertified vertices
                    else predicate = true;        // Active <- impacted vertices (l.15)
                    continue;
                }
                break;
            }
            if (pull) {  // NEXT-1: one pull sweep, then push from the vertices it changed (masks in M)
                relax_pull<KIND, PACKED, L>(P, count, E, xs, n_edges, n_upd, n_read);
                pull = false;
                bits = false;
            } else if (phase == 1 && P.pl_thr != 0u && E >= P.pl_thr) {  // dense phase-1 iteration: pull
                if constexpr (!InitOf<L>::ALL_ACTIVE) relax_pull_all<KIND, PACKED, L>(P, xs, vs, n_edges, n_upd, n_read);
                bits = false;  // the pull marks the next frontier in M
            } else {
                // small frontier: its S2 sets frontier bits (few reds) and the next S1 reads the
                // bitmap; large frontier: no bitmap reds (they contend in L2), the next S1 scans M
                bits = E < P.bits_below;  // at most E vertices change
                relax_b<KIND, PACKED, L>(P, g, count, E, xs, vs, bits, fresh, n_edges, n_upd, n_read,
                                         P.dyn ? ctr + CT_TILE : nullptr);
                predicate = false;
            }
            if (P.trace_cta && tr + 1 < P.trace_cap) {  // S2 load balance across CTAs (trace only)
                __syncthreads();
                if (threadIdx.x == 0) {
                    const unsigned long long tn = global_ns();
                    atomicMin(P.trace_cta + 2ull * tr, tn);
                    atomicMax(P.trace_cta + 2ull * tr + 1, tn);
                }
            }
            grid_sync(P.ctrl, epoch);
            if (P.trace && tid == 0 && tr + 1 < P.trace_cap) P.trace[5ull * tr + 2] = global_ns();
            if (++iters > P.max_iters) {  // cannot happen for a monotone fixpoint; every CTA agrees
                if (tid == 0) report_sticky(P.err_map, sm_err | ERR_ITERS);
                return;
            }
        }
        if (kt && q0 == 0) kt[2] = global_ns();
        if constexpr (KIND == CG_VITERBI || KIND == CG_WCC) {  // u32 only (the host rejects the others)
            transpose_out<L>(P, static_cast<uint32_t*>(P.out), q0, nq, xs, vs);
        } else {
            if (P.out_fmt == CG_OUT_U32) transpose_out<L>(P, static_cast<uint32_t*>(P.out), q0, nq, xs, vs);
            else transpose_narrow<L>(P, q0, nq, xs, vs);
        }
        if (P.stats) {  // reached / precise per query (the thread's query q is fixed)
            grid_sync(P.ctrl, epoch);  // every CTA's values written: the phase-2 end time
            if (tid == 0) sm_t[3] = global_ns();
            const uint32_t q = (uint32_t)(tid % Q);
            const uint32_t sb = ((int)q < nq && P.srcs) ? __ldg(P.srcs + q0 + q) : 0xffffffffu;
            const uint32_t init = L::decode(L::init_word(), 0);
            unsigned long long r = 0, pr = 0;
            if ((int)q < nq)
                for (uint64_t v = tid / Q; v < P.n; v += nthreads / Q) {
                    const uint32_t fv = value_of<L>(P.V, (uint32_t)v, q);
                    if (v != sb && fv != init) {
                        ++r;
                        if (P.p1 && ld_cg(P.p1 + (size_t)(q0 + q) * P.n + v) == fv) ++pr;
                    }
                }
            per_query_add<Q>(P.stats, q0, nq, ST_REACH, r);
            per_query_add<Q>(P.stats, q0, nq, ST_PREC, pr);
        }
        grid_sync(P.ctrl, epoch);  // V / M / bitmap are reused by the next batch
        if (P.stats && tid == 0) {  // device time of this pass's phases, for each of its queries
            for (int b = 0; b < nq; ++b) {
                atomicAdd(P.stats + (size_t)(q0 + b) * NSTAT + ST_T1, sm_t[1] - sm_t[0]);
                atomicAdd(P.stats + (size_t)(q0 + b) * NSTAT + ST_T2, sm_t[3] - sm_t[2]);
            }
        }
    }
    if (kt) kt[3] = global_ns();
    // sticky errors: a bad source (seen by every thread), a narrow-output overflow (any thread,
    // collected in P.err; the pass's final grid barrier made it visible)
    if (tid == 0) report_sticky(P.err_map, sm_err | (ld_cg(P.err) & ERR_NARROW));
}

template <int KIND, bool PACKED, int LW>
void launch_b(const BParams& P, int sms, cudaStream_t s) {
    using L = typename LanesOf<LW, KIND>::T;
    // the certificates' source hub values (sh) only when the call uses them: shared memory not
    // allocated stays L1
    const size_t base = (size_t)BW * (xs_words<L>() + vs_words<L>()) * sizeof(uint32_t);
    constexpr bool HUBS = L::QPW == 1 && L::RW > 1;  // u32 lanes: the only ones given hub certificates
    const size_t smax = base + (HUBS ? (size_t)L::Q * 2 * 64 * sizeof(uint32_t) : 0u);
    const size_t smem = P.HB ? smax : base;
    static int bps = 0;
    if (!bps) {
        if (smax > 48 * 1024)
            CGB_CUDA(cudaFuncSetAttribute(batch_kernel<KIND, PACKED, L>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                          (int)smax));
        CGB_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&bps, batch_kernel<KIND, PACKED, L>, BT, smax));
        CGB_CHECK(bps > 0, CG_EUNSUPPORTED, "batch kernel cannot be resident");
    }
    void* args[] = {(void*)&P};
    CGB_CUDA(cudaLaunchCooperativeKernel((const void*)batch_kernel<KIND, PACKED, L>, dim3(bps * sms), dim3(BT), args,
                                         smem, s));
    count_launch();
}

template <bool PACKED>
void launch_kind_b(int kind, int lw, const BParams& P, int sms, cudaStream_t s) {
    switch (kind) {
    case CG_SSSP:
        if (lw == 16) launch_b<CG_SSSP, PACKED, 16>(P, sms, s);
        else launch_b<CG_SSSP, PACKED, 32>(P, sms, s);
        break;
    case CG_SSWP:
        if (lw == 16) launch_b<CG_SSWP, PACKED, 16>(P, sms, s);
        else launch_b<CG_SSWP, PACKED, 32>(P, sms, s);
        break;
    case CG_SSNP:
        if (lw == 16) launch_b<CG_SSNP, PACKED, 16>(P, sms, s);
        else launch_b<CG_SSNP, PACKED, 32>(P, sms, s);
        break;
    case CG_VITERBI:
        if (lw == 33) launch_b<CG_VITERBI, PACKED, 33>(P, sms, s);
        else launch_b<CG_VITERBI, PACKED, 32>(P, sms, s);
        break;
    case CG_BFS:
        if (lw == 16) launch_b<CG_BFS, PACKED, 16>(P, sms, s);
        else launch_b<CG_BFS, PACKED, 32>(P, sms, s);
        break;
    case CG_REACH:
        if (lw == 1) launch_b<CG_REACH, PACKED, 1>(P, sms, s);
        else launch_b<CG_REACH, PACKED, 32>(P, sms, s);
        break;
    case CG_WCC: launch_b<CG_WCC, PACKED, 2>(P, sms, s); break;
    default: throw Error(CG_EINVAL, "bad kind");
    }
}

// Value lanes of a call: f16 for SSSP / SSWP / SSNP / BFS (SSWP / SSNP need w_max <= 2048, SSSP
// w_max <= 2048; SSSP / BFS fall back to u32 lanes on a lane overflow), one bit for REACH, u32
// for Viterbi (CG_LANES=32 forces u32 lanes for every kind).
int lane_width(const Graph& G, int kind) {
    const char* e = getenv("CG_LANES");
    if (kind == CG_WCC) return 2;  // labels
    if (e && atoi(e) == 32) return 32;
    if (kind == CG_REACH) return 1;
    if (kind == CG_VITERBI) return (e && atoi(e) == 33) ? 33 : 32;  // CG_LANES=33: 32 per pass (measured slower)
    if (kind == CG_BFS) return 16;
    if ((kind == CG_SSSP || kind == CG_SSWP || kind == CG_SSNP) && G.w_max <= 2048) return 16;
    return 32;
}

// One launch of the batched kernel for the call.  guard != null: the u32-lane re-run of a
// binary16 call, which executes only if that call set ERR_LANE_OVERFLOW in *guard (the per-call
// word is then not cleared).
void run_batched_lw(Graph& G, const QueryCall& c, int lw, cudaStream_t s, std::vector<cg_stats>* stats,
                    const uint32_t* guard) {
    BatchSpace& w = G.bs;
    const uint32_t words = (G.n + 31) / 32;
    if (w.n != G.n) {
        w.V.alloc((size_t)G.n * 32, s);  // the widest row: 32 u32 words (Viterbi, 32 per pass)
        w.M.alloc(G.n ? G.n : 1, s);
        w.bitmap.alloc(words ? words : 1, s);
        w.lv.alloc(G.n ? G.n : 1, s);
        w.lo.alloc(G.n ? G.n : 1, s);
        w.lm.alloc(G.n ? G.n : 1, s);
        w.ctrl.alloc(CT0 + CTS * 4, s);
        w.err.alloc(1, s);
        w.n = G.n;
        w.B = 16;
    }
    const int Q = lw == 2 ? 1 : lw == 32 ? 16 : 32;  // (lw 33: u32 lanes, 32 per pass; lw 2: WCC labels)
    DevBuf<unsigned long long> st;
    if (stats) st.alloc((size_t)c.n_src * NSTAT, s);
    BParams P{};
    P.n = G.n;
    P.words = words;
    P.dbits = G.dbits;
    P.dmask = G.dbits >= 32 ? 0xffffffffu : ((1u << G.dbits) - 1u);
    P.G = c.full;
    P.C = c.two_phase ? c.core : c.full;
    P.R = view(G.gr);
    {   // NEXT-1 (Reduced(E) pull) after phase 1 for the kinds with a certificate; CG_REDUCED is a
        // bitmask over cg_kind.  Default REACH only: its certificate (reached = final) leaves only
        // unreachable vertices; the SSWP / SSNP / SSSP certificates (u32 lanes) are exact but,
        // united over a 16-query batch, leave ~99 % of the vertices uncertified for some query
        // (measured, C2).
        const char* e = getenv("CG_REDUCED");
        const unsigned mask = e ? (unsigned)strtoul(e, nullptr, 0) : (1u << CG_REACH);
        const Core& core = G.core[core_slot(c.kind)];
        const bool kind_cg = c.two_phase && c.cg == &core;
        const bool hub_cert = lw == 32 && core.hub_k > 0 && core.hub_k <= 64 && core.hub_vals.get();
        const bool has_cert = c.kind == CG_REACH || hub_cert;
        P.reduced = kind_cg && ((mask >> c.kind) & 1u) && has_cert;
        const char* dy = getenv("CG_DYN");
        P.dyn = dy ? atoi(dy) : 1;
        const char* rs = getenv("CG_REST");
        P.Rst = GraphView{};
        if (c.two_phase && c.rest.ptr && (rs ? atoi(rs) : 1)) P.Rst = c.rest;
        if (P.reduced && c.kind != CG_REACH) {
            P.HB = core.hub_vals.get();
            P.K = core.hub_k;
            P.KP = (core.hub_k + 3) & ~3u;
        }
    }
    {   // phase-1 pull (relax_pull_all) over the kind's CG^R: iterations whose push would scan at
        // least m_cg / CG_PULL_DIV edges (CG_PULL_DIV=0 disables it).  Default: REACH's bit lanes
        // only — measured on C2 (profiles/r2_pull_experiments.txt): with 64 B value rows the
        // segmented scan over 16 row words costs more than the atomics it saves (REACH 0.76 ->
        // 0.69 ms; SSSP 2.53 -> 3.21 ms)
        const char* e = getenv("CG_PULL_DIV");
        const uint32_t div = e ? (uint32_t)strtoul(e, nullptr, 10) : (lw == 1 ? 2u : 0u);
        P.pl_thr = 0;
        if (c.two_phase && c.cg && div && c.cg->rcg_built && c.kind != CG_WCC) {
            const Core& C = *c.cg;
            P.RC = view(C.rcg);
            P.pl_v = C.pl_v.get();
            P.pl_lo = C.pl_lo.get();
            P.pl_count = C.pl_count;
            P.pl_E = C.rcg.m;
            P.pl_thr = C.rcg.m / div > 0 ? C.rcg.m / div : 1u;
        }
    }
    P.srcs = c.srcs;
    P.n_src = c.n_src;
    P.two_phase = c.two_phase;
    P.out = c.out;
    P.out_fmt = c.out_fmt;
    P.p1 = c.two_phase ? c.p1 : nullptr;
    P.V = w.V.get();
    P.M = w.M.get();
    P.bitmap = w.bitmap.get();
    P.lv = w.lv.get();
    P.lo = w.lo.get();
    P.lm = w.lm.get();
    P.ctrl = w.ctrl.get();
    P.stats = stats ? st.get() : nullptr;
    P.err = w.err.get();
    P.err_map = G.sticky_d;
    P.guard = guard;
    P.max_iters = G.n + 8;
    {
        const char* e = getenv("CG_BITS_BELOW");
        P.bits_below = e ? (uint32_t)strtoul(e, nullptr, 10) : G.n / 256;
        const char* f = getenv("CG_FRESH");
        P.fresh = f ? (uint32_t)strtoul(f, nullptr, 10) : 2u;  // phase 2 gathers bypass L1 (measured +1 %; L1 hit rate ~4 %)
    }
    CGB_CUDA(cudaMemsetAsync(w.bitmap.get(), 0, w.bitmap.bytes(), s));
    CGB_CUDA(cudaMemsetAsync(w.ctrl.get(), 0, w.ctrl.bytes(), s));
    if (!guard) CGB_CUDA(cudaMemsetAsync(w.err.get(), 0, 4, s));
    if (stats) CGB_CUDA(cudaMemsetAsync(st.get(), 0, st.bytes(), s));
    static const bool tracing = getenv("CG_TRACE") != nullptr;
    DevBuf<unsigned long long> trace, trace_cta;
    P.trace_cta = nullptr;
    if (tracing) {
        P.trace_cap = 1u << 16;
        trace.alloc(5ull * P.trace_cap, s);
        CGB_CUDA(cudaMemsetAsync(trace.get(), 0, trace.bytes(), s));
        P.trace = trace.get();
        trace_cta.alloc(2ull * P.trace_cap, s);
        std::vector<unsigned long long> init(2ull * P.trace_cap);
        for (size_t i = 0; i < init.size(); i += 2) init[i] = ~0ull, init[i + 1] = 0ull;
        CGB_CUDA(cudaMemcpyAsync(trace_cta.get(), init.data(), trace_cta.bytes(), cudaMemcpyHostToDevice, s));
        CGB_CUDA(cudaStreamSynchronize(s));
        P.trace_cta = trace_cta.get();
    }
    if (G.packed) launch_kind_b<true>(c.kind, lw, P, G.num_sms, s);
    else launch_kind_b<false>(c.kind, lw, P, G.num_sms, s);
    if (tracing) {
        std::vector<unsigned long long> h(5ull * P.trace_cap), hc(2ull * P.trace_cap);
        CGB_CUDA(cudaMemcpyAsync(h.data(), trace.get(), trace.bytes(), cudaMemcpyDeviceToHost, s));
        CGB_CUDA(cudaMemcpyAsync(hc.data(), trace_cta.get(), trace_cta.bytes(), cudaMemcpyDeviceToHost, s));
        CGB_CUDA(cudaStreamSynchronize(s));
        unsigned long long t0 = 0;
        {
            const unsigned long long* k = h.data() + 5ull * (P.trace_cap - 1);
            fprintf(stderr, "CG_TRACE_KERNEL kind=%d Q=%d lanes=%d init+seeds=%.1f batch0_loop_end=%.1f exit=%.1f us\n",
                    c.kind, Q, lw, (k[1] - k[0]) / 1e3, (k[2] - k[0]) / 1e3, (k[3] - k[0]) / 1e3);
        }
        for (uint32_t i = 0; i < P.trace_cap - 1 && h[5 * i]; ++i) {
            const unsigned long long* t = h.data() + 5 * i;
            if (!t0) t0 = t[0];
            fprintf(stderr, "CG_TRACE kind=%d Q=%d lanes=%d it=%u q0=%llu phase=%llu list=%llu active=%llu edges=%llu "
                    "t=%.1f s1=%.1f s2=%.1f us s2_cta_first=%.1f s2_cta_last=%.1f\n", c.kind, Q, lw, i,
                    (t[3] >> 32) & 0x3fffffffull, t[3] >> 62, t[3] & 0xffffffffull, t[4] >> 32, t[4] & 0xffffffffull,
                    (t[0] - t0) / 1e3, (t[1] - t[0]) / 1e3, t[2] ? (t[2] - t[1]) / 1e3 : 0.0,
                    hc[2 * i + 1] ? ((double)hc[2 * i] - (double)t[1]) / 1e3 : 0.0,
                    hc[2 * i + 1] ? ((double)hc[2 * i + 1] - (double)t[1]) / 1e3 : 0.0);
        }
    }
    if (stats) {
        std::vector<unsigned long long> h((size_t)c.n_src * NSTAT);
        CGB_CUDA(cudaMemcpyAsync(h.data(), st.get(), st.bytes(), cudaMemcpyDeviceToHost, s));
        CGB_CUDA(cudaStreamSynchronize(s));
        stats->resize(c.n_src);
        for (int qq = 0; qq < c.n_src; ++qq) {
            const unsigned long long* x = h.data() + (size_t)qq * NSTAT;
            cg_stats& o = (*stats)[qq];
            o.iters_p1 = (int64_t)x[ST_IT1];
            o.iters_p2 = (int64_t)x[ST_IT2];
            o.edges_p1 = (int64_t)x[ST_E1];
            o.edges_p2 = (int64_t)x[ST_E2];
            o.updates_p1 = (int64_t)x[ST_U1];
            o.updates_p2 = (int64_t)x[ST_U2];
            o.frontier_p1 = (int64_t)x[ST_F1];
            o.frontier_p2 = (int64_t)x[ST_F2];
            o.impacted = (int64_t)x[ST_IMP];
            o.reached = (int64_t)x[ST_REACH];
            o.precise_p1 = P.p1 ? (int64_t)x[ST_PREC] : -1;
            o.scanned_p1 = (int64_t)x[ST_S1];
            o.scanned_p2 = (int64_t)x[ST_S2];
            o.batch_queries = Q;
            o.row_bytes = (lw == 1 || lw == 2) ? 4 : lw == 33 ? 128 : 64;
            o.ms_p1 = (float)(x[ST_T1] * 1e-6);
            o.ms_p2 = (float)(x[ST_T2] * 1e-6);
        }
    }
}

}  // namespace

int pass_width(const Graph& G, int kind) {  // queries one batched-engine pass evaluates together
    if (!batch_width()) return 1;
    const int lw = lane_width(G, kind);
    return lw == 2 ? 1 : lw == 32 ? 16 : 32;
}

int batch_width() {
    const char* e = getenv("CG_BATCH");
    return (e && atoi(e) == 0) ? 0 : 16;  // CG_BATCH=0: single-query engine (engine.cu)
}

void run_queries_batched(Graph& G, const QueryCall& c, int, cudaStream_t s, std::vector<cg_stats>* stats) {
    const int lw = lane_width(G, c.kind);
    run_batched_lw(G, c, lw, s, stats, nullptr);
    // binary16 SSSP / BFS lanes (reading N3) raise ERR_LANE_OVERFLOW when a candidate reaches
    // 2048; the call is then re-run with u32 lanes.  Without stats the re-run is enqueued
    // unconditionally and exits at once unless the flag is set (no host synchronisation, so the
    // call stays asynchronous and capturable); with stats the call synchronises anyway.
    if (lw == 16 && (c.kind == CG_BFS || c.kind == CG_SSSP)) {
        if (stats) {
            uint32_t* err = G.bs.err_host();
            CGB_CUDA(cudaMemcpyAsync(err, G.bs.err.get(), 4, cudaMemcpyDeviceToHost, s));
            CGB_CUDA(cudaStreamSynchronize(s));
            if (*err & ERR_LANE_OVERFLOW) run_batched_lw(G, c, 32, s, stats, nullptr);
        } else {
            run_batched_lw(G, c, 32, s, nullptr, G.bs.err.get());
        }
    }
}

}  // namespace cgb
