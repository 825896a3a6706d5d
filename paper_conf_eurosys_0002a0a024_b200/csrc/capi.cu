// capi.cu — the extern "C" boundary declared in include/cg.h.  Argument checking, error
// translation (no exception crosses the ABI), allocator plumbing, and the host-buffer
// end-to-end query path.  All compute happens in the kernels of the other .cu files.
#include <cstring>
#include <mutex>
#include <string>
#include <vector>

#include "graph.hpp"

namespace cgb {

std::atomic<int64_t> g_launches{0};

namespace {
cg_alloc_fn g_alloc = nullptr;
cg_free_fn g_free = nullptr;
void* g_ctx = nullptr;
thread_local std::string g_err;
}  // namespace

void* dev_alloc(size_t bytes, cudaStream_t s) {
    if (!bytes) return nullptr;
    void* p = nullptr;
    if (g_alloc) {
        p = g_alloc(bytes, (void*)s, g_ctx);
        if (!p) throw Error(CG_ENOMEM, "allocator callback failed for " + std::to_string(bytes) + " bytes");
        return p;
    }
    cudaError_t e = cudaMalloc(&p, bytes);
    if (e != cudaSuccess) {
        cudaGetLastError();
        throw Error(CG_ENOMEM, "cudaMalloc(" + std::to_string(bytes) + "): " + cudaGetErrorString(e));
    }
    return p;
}

void dev_free(void* p, cudaStream_t s) {
    if (!p) return;
    if (g_free) g_free(p, (void*)s, g_ctx);
    else {
        cudaStreamSynchronize(s);
        cudaFree(p);
    }
}

}  // namespace cgb

using namespace cgb;

struct cg_graph_s {
    Graph G;
    cudaStream_t stream = nullptr;  // stream the graph's memory was allocated on
};

namespace capi_internal {

template <typename F>
cg_status guard(F&& f) {
    try {
        f();
        return CG_OK;
    } catch (const Error& e) {
        g_err = e.what();
        return e.code;
    } catch (const std::bad_alloc&) {
        g_err = "host allocation failed";
        return CG_ENOMEM;
    } catch (const std::exception& e) {
        g_err = e.what();
        return CG_EINTERNAL;
    } catch (...) {
        g_err = "unknown exception";
        return CG_EINTERNAL;
    }
}

inline cudaStream_t S(void* s) { return (cudaStream_t)s; }

void check_kind(int kind) { CGB_CHECK(kind >= CG_SSSP && kind <= CG_WCC, CG_EINVAL, "bad cg_kind"); }

void check_sources_host(const Graph& G, const uint32_t* src, int32_t n_src) {
    for (int32_t i = 0; i < n_src; ++i) CGB_CHECK(src[i] < G.n, CG_EINVAL, "source id >= n");
}

// the graph's sticky device error (graph.hpp), returned (and cleared) by the next call
void take_sticky(Graph& G) {
    if (!G.sticky_h) return;
    volatile uint32_t* p = G.sticky_h;
    const uint32_t e = *p;
    if (!e) return;
    *p = 0u;
    CGB_CHECK(!(e & ERR_SOURCE), CG_EINVAL, "a source id >= n was passed to an asynchronous query (its row holds InitVal)");
    CGB_CHECK(!(e & ERR_NARROW), CG_EOVERFLOW, "a value did not fit the requested narrow output format");
    CGB_CHECK(!(e & ERR_ITERS), CG_EINTERNAL, "iteration bound exceeded");
}

// calls on one graph run in issue order across streams (they share the workspace)
void order_begin(Graph& G, cudaStream_t s) {
    if (G.last_valid && G.last_stream != s) CGB_CUDA(cudaStreamWaitEvent(s, G.last, 0));
}
void order_end(Graph& G, cudaStream_t s) {
    CGB_CUDA(cudaEventRecord(G.last, s));
    G.last_stream = s;
    G.last_valid = true;
}

size_t row_bytes_of(const Graph& G, int fmt) {
    return fmt == CG_OUT_U16 ? 2ull * G.n : fmt == CG_OUT_BITS ? 4ull * ((G.n + 31) / 32) : 4ull * G.n;
}

void check_format(int kind, int fmt) {
    CGB_CHECK(fmt == CG_OUT_U32 || fmt == CG_OUT_U16 || fmt == CG_OUT_BITS, CG_EINVAL, "bad cg_out_format");
    CGB_CHECK(fmt != CG_OUT_U16 || (kind != CG_VITERBI && kind != CG_WCC), CG_EINVAL,
              "CG_OUT_U16 holds integer values: not for VITERBI or WCC");
    CGB_CHECK(fmt != CG_OUT_BITS || kind == CG_REACH, CG_EINVAL, "CG_OUT_BITS is REACH's format");
}

void prepare_query(cg_graph g, int kind, int32_t n_src, int mode, const void* out, const uint32_t* src) {
    CGB_CHECK(g != nullptr, CG_EINVAL, "null graph");
    take_sticky(g->G);
    check_kind(kind);
    CGB_CHECK(n_src >= 0, CG_EINVAL, "n_src < 0");
    CGB_CHECK(mode == CG_MODE_2PHASE || mode == CG_MODE_FULL, CG_EINVAL, "bad cg_mode");
    CGB_CHECK(n_src == 0 || (out && (src || kind == CG_WCC)), CG_EINVAL, "null src/out");
    CGB_CHECK(kind != CG_WCC || n_src <= 1, CG_EINVAL, "CG_WCC is a whole-graph query: n_src must be 1");
    if (kind == CG_SSSP)
        CGB_CHECK((uint64_t)(g->G.n - 1) * g->G.w_max < 0xFFFFFFFFull, CG_EOVERFLOW,
                  "(n-1)*w_max >= 2^32-1: SSSP distances could wrap");
    if (mode == CG_MODE_2PHASE)
        CGB_CHECK(g->G.core[core_slot(kind)].built, CG_ENOCG, "cg_build has not been called for this kind");
}

}  // namespace capi_internal

using namespace capi_internal;

extern "C" {

cg_status cg_set_allocator(cg_alloc_fn alloc, cg_free_fn free_fn, void* ctx) {
    return guard([&] {
        CGB_CHECK((alloc == nullptr) == (free_fn == nullptr), CG_EINVAL, "alloc and free must both be set or NULL");
        g_alloc = alloc;
        g_free = free_fn;
        g_ctx = ctx;
    });
}

cg_status cg_graph_create(int device, int64_t n, int64_t m, const uint32_t* src, const uint32_t* dst,
                          const uint32_t* w, void* stream, cg_graph* out) {
    return guard([&] {
        CGB_CHECK(out != nullptr, CG_EINVAL, "null out");
        *out = nullptr;
        CGB_CHECK(n > 0, CG_EINVAL, "n must be > 0");
        CGB_CHECK(m >= 0, CG_EINVAL, "m must be >= 0");
        CGB_CHECK(m == 0 || (src && dst && w), CG_EINVAL, "null edge array");
        CGB_CUDA(cudaSetDevice(device));
        int coop = 0;
        CGB_CUDA(cudaDeviceGetAttribute(&coop, cudaDevAttrCooperativeLaunch, device));
        CGB_CHECK(coop, CG_EUNSUPPORTED, "device does not support cooperative launch");
        auto* h = new cg_graph_s();
        try {
            h->G.device = device;
            h->stream = S(stream);
            CGB_CUDA(cudaDeviceGetAttribute(&h->G.num_sms, cudaDevAttrMultiProcessorCount, device));
            CGB_CUDA(cudaHostAlloc(&h->G.sticky_h, sizeof(uint32_t), cudaHostAllocMapped));
            *h->G.sticky_h = 0u;
            CGB_CUDA(cudaHostGetDevicePointer((void**)&h->G.sticky_d, h->G.sticky_h, 0));
            CGB_CUDA(cudaEventCreateWithFlags(&h->G.last, cudaEventDisableTiming));
            build_graph(h->G, n, m, src, dst, w, S(stream));
        } catch (...) {
            delete h;
            throw;
        }
        *out = h;
    });
}

cg_status cg_graph_destroy(cg_graph g) {
    return guard([&] {
        if (!g) return;
        cudaSetDevice(g->G.device);
        cudaStreamSynchronize(g->stream);
        if (g->G.last_valid) cudaEventSynchronize(g->G.last);
        delete g;
    });
}

cg_status cg_graph_info(cg_graph g, int64_t* n, int64_t* m, uint32_t* w_max) {
    return guard([&] {
        CGB_CHECK(g != nullptr, CG_EINVAL, "null graph");
        if (n) *n = g->G.n;
        if (m) *m = g->G.m;
        if (w_max) *w_max = g->G.w_max;
    });
}

cg_status cg_graph_export(cg_graph g, int transpose, int64_t* ptr, uint32_t* idx, uint32_t* w, void* stream) {
    return guard([&] {
        CGB_CHECK(g != nullptr, CG_EINVAL, "null graph");
        CGB_CHECK(ptr && (idx != nullptr) == (w != nullptr), CG_EINVAL, "null output");
        CGB_CUDA(cudaSetDevice(g->G.device));
        export_adj(g->G, transpose ? g->G.gr : g->G.g, ptr, idx, w, S(stream));
    });
}

cg_status cg_build_ex(cg_graph g, cg_kind kind, int32_t K, cg_hub_policy policy, const uint32_t* hubs, uint64_t seed,
                      cg_cg_alg alg, int32_t connectivity, void* stream) {
    return guard([&] {
        CGB_CHECK(g != nullptr, CG_EINVAL, "null graph");
        check_kind(kind);
        CGB_CUDA(cudaSetDevice(g->G.device));
        if (kind == CG_SSSP)
            CGB_CHECK((uint64_t)(g->G.n - 1) * g->G.w_max < 0xFFFFFFFFull, CG_EOVERFLOW,
                      "(n-1)*w_max >= 2^32-1: SSSP distances could wrap");
        order_begin(g->G, S(stream));
        build_core(g->G, kind, K, policy, hubs, seed, alg, connectivity, S(stream));
        order_end(g->G, S(stream));
    });
}

cg_status cg_build(cg_graph g, cg_kind kind, int32_t K, cg_hub_policy policy, const uint32_t* hubs, uint64_t seed,
                   void* stream) {
    return cg_build_ex(g, kind, K, policy, hubs, seed, CG_ALG_AUTO, -1, stream);
}

cg_status cg_build_partial(cg_graph g, cg_kind kind, int32_t K, cg_hub_policy policy, const uint32_t* hubs,
                           uint64_t seed, int32_t hub_begin, int32_t hub_end, uint8_t* flags, void* stream) {
    return guard([&] {
        CGB_CHECK(g != nullptr && (flags != nullptr || g->G.m == 0), CG_EINVAL, "null argument");
        check_kind(kind);
        CGB_CUDA(cudaSetDevice(g->G.device));
        order_begin(g->G, S(stream));
        build_core_partial(g->G, kind, K, policy, hubs, seed, hub_begin, hub_end, flags, S(stream));
        order_end(g->G, S(stream));
    });
}

cg_status cg_build_from_flags(cg_graph g, cg_kind kind, int32_t K, cg_hub_policy policy, const uint32_t* hubs,
                              uint64_t seed, const uint8_t* flags, int32_t connectivity, void* stream) {
    return guard([&] {
        CGB_CHECK(g != nullptr && (flags != nullptr || g->G.m == 0), CG_EINVAL, "null argument");
        check_kind(kind);
        CGB_CUDA(cudaSetDevice(g->G.device));
        order_begin(g->G, S(stream));
        build_core_from_flags(g->G, kind, K, policy, hubs, seed, flags, connectivity, S(stream));
        order_end(g->G, S(stream));
    });
}

cg_status cg_core_save(cg_graph g, cg_kind kind, const char* path, void* stream) {
    return guard([&] {
        CGB_CHECK(g != nullptr && path != nullptr, CG_EINVAL, "null argument");
        check_kind(kind);
        CGB_CUDA(cudaSetDevice(g->G.device));
        order_begin(g->G, S(stream));
        save_core(g->G, kind, path, S(stream));
        order_end(g->G, S(stream));
    });
}

cg_status cg_core_load(cg_graph g, cg_kind kind, const char* path, void* stream) {
    return guard([&] {
        CGB_CHECK(g != nullptr && path != nullptr, CG_EINVAL, "null argument");
        check_kind(kind);
        CGB_CUDA(cudaSetDevice(g->G.device));
        order_begin(g->G, S(stream));
        load_core(g->G, kind, path, S(stream));
        order_end(g->G, S(stream));
    });
}

cg_status cg_core_info(cg_graph g, cg_kind kind, int64_t* m_cg, int32_t* K, uint32_t* hubs, float* build_ms) {
    return guard([&] {
        CGB_CHECK(g != nullptr, CG_EINVAL, "null graph");
        check_kind(kind);
        const Core& C = g->G.core[core_slot(kind)];
        CGB_CHECK(C.built, CG_ENOCG, "Core Graph not built for this kind");
        if (m_cg) *m_cg = C.m_cg;
        if (K) *K = (int32_t)C.hubs.size();
        if (hubs) std::memcpy(hubs, C.hubs.data(), 4 * C.hubs.size());
        if (build_ms) *build_ms = C.build_ms;
    });
}

cg_status cg_core_export(cg_graph g, cg_kind kind, uint8_t* flags, void* stream) {
    return guard([&] {
        CGB_CHECK(g != nullptr && flags != nullptr, CG_EINVAL, "null argument");
        check_kind(kind);
        const Core& C = g->G.core[core_slot(kind)];
        CGB_CHECK(C.built, CG_ENOCG, "Core Graph not built for this kind");
        CGB_CUDA(cudaSetDevice(g->G.device));
        export_core_flags(g->G, C, flags, S(stream));
    });
}

}  // extern "C"

namespace capi_internal {

// the call's engine inputs: G (split rows of the kind's CG in 2Phase), CG, G minus CG
QueryCall make_call(Graph& G, int kind, bool two, const uint32_t* src, int32_t n_src, void* out, uint32_t* p1,
                    bool want_stats, int fmt) {
    QueryCall c{};
    c.kind = kind;
    c.two_phase = two ? 1 : 0;
    c.srcs = src;
    c.n_src = n_src;
    c.out = out;
    c.p1 = two ? p1 : nullptr;
    c.want_stats = want_stats;
    c.out_fmt = fmt;
    if (kind == CG_WCC) {  // G ∪ G^R, CG ∪ CG^R
        c.full = view(G.gsym);
        c.core = two ? view(G.core[CG_REACH].sym) : c.full;
        c.rest = GraphView{};
        c.cg = nullptr;
        return c;
    }
    const Core& C = G.core[core_slot(kind)];
    if (two) {
        c.full = split_view(G, C);
        c.core = core_view(G, C);
        c.rest = rest_view(G, C);
        c.cg = &C;
    } else {
        c.full = view(G.g);
        c.core = c.full;
        c.rest = GraphView{};
        c.cg = nullptr;
    }
    return c;
}

}  // namespace capi_internal

extern "C" {

cg_status cg_query_fmt(cg_graph g, cg_kind kind, const uint32_t* src, int32_t n_src, cg_mode mode, cg_out_format fmt,
                       void* out, void* p1_out, cg_stats* stats, void* stream) {
    return guard([&] {
        prepare_query(g, kind, n_src, mode, out, src);
        check_format(kind, fmt);
        if (n_src == 0) return;
        Graph& G = g->G;
        CGB_CUDA(cudaSetDevice(G.device));
        cudaStream_t s = S(stream);
        order_begin(G, s);
        if (kind == CG_WCC) src = nullptr;  // whole-graph query: no source
        if (kind == CG_WCC) ensure_wcc_graphs(G, mode == CG_MODE_2PHASE, s);
        const bool two = mode == CG_MODE_2PHASE;
        QueryCall c = make_call(G, kind, two, src, n_src, out, (uint32_t*)p1_out, stats != nullptr, fmt);
        std::vector<cg_stats> st;
        run_queries(G, c, s, stats ? &st : nullptr);
        order_end(G, s);
        if (stats) {
            CGB_CUDA(cudaStreamSynchronize(s));
            take_sticky(G);  // this call's own device errors
            std::memcpy(stats, st.data(), sizeof(cg_stats) * (size_t)n_src);
        }
    });
}

cg_status cg_query_ex(cg_graph g, cg_kind kind, const uint32_t* src, int32_t n_src, cg_mode mode, void* out,
                      void* p1_out, cg_stats* stats, void* stream) {
    return cg_query_fmt(g, kind, src, n_src, mode, CG_OUT_U32, out, p1_out, stats, stream);
}

cg_status cg_query(cg_graph g, cg_kind kind, const uint32_t* src, int32_t n_src, cg_mode mode, void* out,
                   cg_stats* stats, void* stream) {
    return cg_query_fmt(g, kind, src, n_src, mode, CG_OUT_U32, out, nullptr, stats, stream);
}

cg_status cg_graph_status(cg_graph g, void* stream) {
    return guard([&] {
        CGB_CHECK(g != nullptr, CG_EINVAL, "null graph");
        CGB_CUDA(cudaSetDevice(g->G.device));
        CGB_CUDA(cudaStreamSynchronize(S(stream)));
        if (g->G.hp.cp) CGB_CUDA(cudaStreamSynchronize(g->G.hp.cp));  // asynchronous host calls' result copies
        take_sticky(g->G);
    });
}

// The host path (cg_query_host*): sources host -> device, the queries in device batches of `batch`,
// each batch's rows device -> host on the graph's copy stream while the next batch computes.  The
// result slots, the device sources and the copy stream persist in the graph (HostPath), so an
// asynchronous call returns with its copies still in flight and the NEXT call (another kind, say)
// computes while they drain; slot reuse is ordered by events (done / drained), across calls too.
// At the end the call's stream waits for its last copy: synchronising `stream` completes `out`.
static void query_host(cg_graph g, cg_kind kind, const uint32_t* src, int32_t n_src, cg_mode mode, cg_out_format fmt,
                       void* out, int32_t batch, void* stream, bool sync) {
    prepare_query(g, kind, n_src, mode, out, src);
    check_format(kind, fmt);
    if (n_src == 0) return;
    Graph& G = g->G;
    if (kind == CG_WCC) src = nullptr;
    if (src) check_sources_host(G, src, n_src);
    CGB_CUDA(cudaSetDevice(G.device));
    cudaStream_t s = S(stream);
    order_begin(G, s);
    if (kind == CG_WCC) ensure_wcc_graphs(G, mode == CG_MODE_2PHASE, s);
    const size_t row = row_bytes_of(G, fmt);
    if (batch <= 0) {  // ~512 MiB of results per batch, rounded down to whole engine passes, at least 1 query
        size_t b = ((size_t)512 << 20) / (row ? row : 1);
        const size_t pw = (size_t)pass_width(G, kind);
        if (b >= pw) b -= b % pw;
        batch = (int32_t)(b < 1 ? 1 : (b > (size_t)n_src ? (size_t)n_src : b));
    }
    if (batch > n_src) batch = n_src;
    HostPath& h = G.hp;
    if (!h.cp) {
        CGB_CUDA(cudaStreamCreateWithFlags(&h.cp, cudaStreamNonBlocking));
        for (int i = 0; i < 2; ++i) {
            CGB_CUDA(cudaEventCreateWithFlags(&h.done[i], cudaEventDisableTiming));
            CGB_CUDA(cudaEventCreateWithFlags(&h.drained[i], cudaEventDisableTiming));
        }
        for (int i = 0; i < 2; ++i) CGB_CUDA(cudaEventCreateWithFlags(&h.src_copied[i], cudaEventDisableTiming));
    }
    const size_t need = (size_t)batch * row;
    for (int k = 0; k < 2; ++k) {
        if (h.slot[k].n >= need) continue;
        if (h.pending[k]) CGB_CUDA(cudaEventSynchronize(h.drained[k]));  // a copy may still read the old slot
        h.slot[k].alloc(need, s);
        h.pending[k] = false;
    }
    if (src) {  // host -> pinned staging (two buffers, alternating) -> device: asynchronous for any src
        const int k = h.src_next;
        h.src_next ^= 1;
        if (h.src_pending[k]) CGB_CUDA(cudaEventSynchronize(h.src_copied[k]));  // that buffer's last copy is done
        h.src_pending[k] = false;
        if (h.hsrc_n[k] < (size_t)n_src) {
            if (h.hsrc[k]) CGB_CUDA(cudaFreeHost(h.hsrc[k]));
            h.hsrc[k] = nullptr;
            h.hsrc_n[k] = 0;
            CGB_CUDA(cudaMallocHost(&h.hsrc[k], 4ull * n_src));
            h.hsrc_n[k] = (size_t)n_src;
        }
        memcpy(h.hsrc[k], src, 4ull * n_src);
        if (h.dsrc.n < (size_t)n_src) h.dsrc.alloc((size_t)n_src, s);  // stream-ordered after its last reader
        CGB_CUDA(cudaMemcpyAsync(h.dsrc.get(), h.hsrc[k], 4ull * n_src, cudaMemcpyHostToDevice, s));
        CGB_CUDA(cudaEventRecord(h.src_copied[k], s));
        h.src_pending[k] = true;
    }
    const bool two = mode == CG_MODE_2PHASE;
    for (int32_t q0 = 0; q0 < n_src; q0 += batch) {
        const int32_t nq = (n_src - q0) < batch ? (n_src - q0) : batch;
        const int k = h.next;
        h.next ^= 1;
        if (h.pending[k]) CGB_CUDA(cudaStreamWaitEvent(s, h.drained[k], 0));  // slot k's previous rows copied out
        QueryCall c = make_call(G, kind, two, src ? h.dsrc.get() + q0 : nullptr, nq, h.slot[k].get(), nullptr, false,
                                fmt);
        run_queries(G, c, s, nullptr);
        CGB_CUDA(cudaEventRecord(h.done[k], s));
        CGB_CUDA(cudaStreamWaitEvent(h.cp, h.done[k], 0));
        CGB_CUDA(cudaMemcpyAsync((uint8_t*)out + (size_t)q0 * row, h.slot[k].get(), (size_t)nq * row,
                                 cudaMemcpyDeviceToHost, h.cp));
        CGB_CUDA(cudaEventRecord(h.drained[k], h.cp));
        h.pending[k] = true;
    }
    order_end(G, s);  // the call's copies complete on h.cp: cg_graph_status / a synchronous call wait for them
    if (sync) {
        CGB_CUDA(cudaStreamSynchronize(s));
        CGB_CUDA(cudaStreamSynchronize(h.cp));
        take_sticky(G);
    }
}

cg_status cg_query_host_fmt(cg_graph g, cg_kind kind, const uint32_t* src, int32_t n_src, cg_mode mode,
                            cg_out_format fmt, void* out, int32_t batch, void* stream) {
    return guard([&] { query_host(g, kind, src, n_src, mode, fmt, out, batch, stream, true); });
}

cg_status cg_query_host_async(cg_graph g, cg_kind kind, const uint32_t* src, int32_t n_src, cg_mode mode,
                              cg_out_format fmt, void* out, int32_t batch, void* stream) {
    return guard([&] { query_host(g, kind, src, n_src, mode, fmt, out, batch, stream, false); });
}

cg_status cg_query_host(cg_graph g, cg_kind kind, const uint32_t* src, int32_t n_src, cg_mode mode, void* out,
                        int32_t batch, void* stream) {
    return cg_query_host_fmt(g, kind, src, n_src, mode, CG_OUT_U32, out, batch, stream);
}

cg_status cg_rmat_generate(uint64_t n, uint32_t tA, uint32_t tAB, uint32_t tABC, uint32_t w_max, uint64_t seed,
                           int32_t permute, uint64_t e0, uint64_t count, uint32_t* src, uint32_t* dst, uint32_t* w,
                           void* stream) {
    return guard([&] { rmat_generate(n, tA, tAB, tABC, w_max, seed, permute, e0, count, src, dst, w, S(stream)); });
}

int64_t cg_kernel_launches(void) { return g_launches.load(); }

const char* cg_status_string(cg_status s) {
    switch (s) {
    case CG_OK: return "CG_OK";
    case CG_EINVAL: return "CG_EINVAL";
    case CG_ENOMEM: return "CG_ENOMEM";
    case CG_ECUDA: return "CG_ECUDA";
    case CG_ENOCG: return "CG_ENOCG";
    case CG_EOVERFLOW: return "CG_EOVERFLOW";
    case CG_EUNSUPPORTED: return "CG_EUNSUPPORTED";
    case CG_EINTERNAL: return "CG_EINTERNAL";
    }
    return "CG_UNKNOWN";
}

const char* cg_last_error(void) { return g_err.c_str(); }

}  // extern "C"
