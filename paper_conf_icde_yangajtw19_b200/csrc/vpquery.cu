// vpquery.cu — the vertex-partitioned search of ONE query driven by the library (SURVEY.md §8(e),
// DESIGN.md "Multi-GPU"): the level loop, the exchanges and the stop rules of Def. 4 / Thm. V.3 / R9 /
// R22, then the top-down on the replicated state.  The ranks' collectives go through a transport
// (kgs_vp_transport): the library's own NCCL communicator (NVLink / NVSwitch on a multi-GPU node), or
// caller callbacks (the CPU gloo tests).  Product code; shares nothing with oracle/.
//
// Per level l (kernels in vpart.cu):  kgs_vp_level (pull over the owned rows)  ->  all_reduce(counts)
//   -> exchange of the owned hit masks: DENSE (all_gather of every rank's slice, n bytes) or, when fewer
//      than n/16 nodes changed in total, SPARSE (all_gather of the per-rank change counts, then of the
//      padded (id << 8 | mask) lists, applied to the replicated masks)
//   -> stop rule: |C| >= k (d = l + 1), max_depth, or exhausted (no mark and no node still waiting for a
//      gated neighbour: kgs_vp_waiting, one more all_reduce).
// After the search: all_gather of the owned M rows and of the central lists, then kgs_vp_topdown.
#include <cuda_runtime.h>
#include <dlfcn.h>

#include <algorithm>
#include <cstring>
#include <string>
#include <vector>

#include "kgs_internal.h"

namespace kgs {
kgs_status set_error(kgs_status s, const std::string &msg);
int64_t graph_nodes(const kgs_graph *g);
int graph_device(const kgs_graph *g);
}  // namespace kgs

using namespace kgs;

namespace {

// ---------------------------------------------------------------- NCCL transport (dlopen: the process's copy)
// The few NCCL entry points the exchange needs, resolved at run time from the libnccl.so.2 already loaded
// in the process (torch's) or else the system's, so that one process never holds two NCCL copies.
typedef int nccl_result;
struct NcclUid { char internal[128]; };
typedef struct ncclComm *ncclComm_t;
enum { kNcclInt8 = 0, kNcclUint8 = 1, kNcclInt64 = 4 };
enum { kNcclSum = 0 };

struct NcclApi {
    void *lib = nullptr;
    nccl_result (*get_unique_id)(NcclUid *) = nullptr;
    nccl_result (*comm_init_rank)(ncclComm_t *, int, NcclUid, int) = nullptr;
    nccl_result (*all_gather)(const void *, void *, size_t, int, ncclComm_t, cudaStream_t) = nullptr;
    nccl_result (*all_reduce)(const void *, void *, size_t, int, int, ncclComm_t, cudaStream_t) = nullptr;
    nccl_result (*comm_destroy)(ncclComm_t) = nullptr;
    const char *(*error_string)(nccl_result) = nullptr;
};

bool nccl_api(NcclApi &a, std::string &why) {
    static NcclApi cached;
    static bool ok = false;
    if (ok) { a = cached; return true; }
    void *h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_NOLOAD);
    if (!h) h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
    if (!h) { why = std::string("libnccl.so.2 not found: ") + dlerror(); return false; }
    NcclApi x;
    x.lib = h;
    x.get_unique_id = reinterpret_cast<decltype(x.get_unique_id)>(dlsym(h, "ncclGetUniqueId"));
    x.comm_init_rank = reinterpret_cast<decltype(x.comm_init_rank)>(dlsym(h, "ncclCommInitRank"));
    x.all_gather = reinterpret_cast<decltype(x.all_gather)>(dlsym(h, "ncclAllGather"));
    x.all_reduce = reinterpret_cast<decltype(x.all_reduce)>(dlsym(h, "ncclAllReduce"));
    x.comm_destroy = reinterpret_cast<decltype(x.comm_destroy)>(dlsym(h, "ncclCommDestroy"));
    x.error_string = reinterpret_cast<decltype(x.error_string)>(dlsym(h, "ncclGetErrorString"));
    if (!x.get_unique_id || !x.comm_init_rank || !x.all_gather || !x.all_reduce || !x.comm_destroy || !x.error_string) {
        why = "libnccl.so.2 lacks an entry point";
        return false;
    }
    cached = x;
    ok = true;
    a = x;
    return true;
}

struct NcclTransport {
    NcclApi api;
    ncclComm_t comm = nullptr;
};

int32_t nccl_all_gather(void *ctx, const void *send, void *recv, int64_t bytes, void *stream) {
    auto *t = static_cast<NcclTransport *>(ctx);
    return t->api.all_gather(send, recv, (size_t)bytes, kNcclUint8, t->comm, (cudaStream_t)stream) == 0 ? 0 : -1;
}
int32_t nccl_all_reduce_i64(void *ctx, int64_t *buf, int64_t count, void *stream) {
    auto *t = static_cast<NcclTransport *>(ctx);
    return t->api.all_reduce(buf, buf, (size_t)count, kNcclInt64, kNcclSum, t->comm, (cudaStream_t)stream) == 0 ? 0 : -1;
}

// The transport's collectives, staged through host memory when the transport asks for it (host_staged:
// the callbacks then see host buffers; the CPU gloo tests).
struct Coll {
    const kgs_vp_transport *t;
    int world;
    cudaStream_t s;
    std::vector<uint8_t> hs, hr;
    int32_t all_gather(const void *send, void *recv, int64_t bytes) {
        if (!t->host_staged) return t->all_gather(t->ctx, send, recv, bytes, (void *)s);
        hs.resize((size_t)std::max<int64_t>(bytes, 1));
        hr.resize((size_t)std::max<int64_t>(bytes * world, 1));
        if (cudaMemcpyAsync(hs.data(), send, (size_t)bytes, cudaMemcpyDeviceToHost, s) != cudaSuccess ||
            cudaStreamSynchronize(s) != cudaSuccess)
            return -1;
        if (t->all_gather(t->ctx, hs.data(), hr.data(), bytes, (void *)s) != 0) return -1;
        return cudaMemcpyAsync(recv, hr.data(), (size_t)(bytes * world), cudaMemcpyHostToDevice, s) == cudaSuccess &&
                       cudaStreamSynchronize(s) == cudaSuccess ? 0 : -1;
    }
    int32_t all_reduce_i64(int64_t *buf, int64_t count) {
        if (!t->host_staged) return t->all_reduce_sum_i64(t->ctx, buf, count, (void *)s);
        hs.resize((size_t)count * sizeof(int64_t));
        if (cudaMemcpyAsync(hs.data(), buf, (size_t)count * sizeof(int64_t), cudaMemcpyDeviceToHost, s) != cudaSuccess ||
            cudaStreamSynchronize(s) != cudaSuccess)
            return -1;
        if (t->all_reduce_sum_i64(t->ctx, reinterpret_cast<int64_t *>(hs.data()), count, (void *)s) != 0) return -1;
        return cudaMemcpyAsync(buf, hs.data(), (size_t)count * sizeof(int64_t), cudaMemcpyHostToDevice, s) == cudaSuccess &&
                       cudaStreamSynchronize(s) == cudaSuccess ? 0 : -1;
    }
};

#define VQ_TRY(expr)                                                                                    \
    do {                                                                                                \
        cudaError_t _e = (expr);                                                                        \
        if (_e != cudaSuccess) {                                                                        \
            st = set_error(_e == cudaErrorMemoryAllocation ? KGS_ENOMEM : KGS_ECUDA,                    \
                           std::string(#expr) + ": " + cudaGetErrorString(_e));                         \
            goto done;                                                                                  \
        }                                                                                               \
    } while (0)
#define VQ_COLL(expr)                                                                                   \
    do {                                                                                                \
        if ((expr) != 0) { st = set_error(KGS_ENCCL, "vertex partition: collective failed: " #expr); goto done; } \
    } while (0)
#define VQ_OK(expr)                                                                                     \
    do {                                                                                                \
        st = (expr);                                                                                    \
        if (st != KGS_OK) goto done;                                                                    \
    } while (0)

}  // namespace

extern "C" {

kgs_status kgs_vp_nccl_unique_id(uint8_t *id) {
    if (!id) return set_error(KGS_EINVAL, "null argument");
    NcclApi a;
    std::string why;
    if (!nccl_api(a, why)) return set_error(KGS_ENCCL, why);
    NcclUid u;
    const nccl_result r = a.get_unique_id(&u);
    if (r != 0) return set_error(KGS_ENCCL, std::string("ncclGetUniqueId: ") + a.error_string(r));
    std::memcpy(id, u.internal, sizeof(u.internal));
    return KGS_OK;
}

kgs_status kgs_vp_nccl_transport(const uint8_t *id, int32_t rank, int32_t world, int32_t device,
                                 kgs_vp_transport *out) {
    if (!id || !out || world < 1 || rank < 0 || rank >= world) return set_error(KGS_EINVAL, "bad transport arguments");
    std::memset(out, 0, sizeof(*out));
    NcclApi a;
    std::string why;
    if (!nccl_api(a, why)) return set_error(KGS_ENCCL, why);
    if (cudaSetDevice(device) != cudaSuccess) return set_error(KGS_ECUDA, "cudaSetDevice");
    auto *t = new NcclTransport();
    t->api = a;
    NcclUid u;
    std::memcpy(u.internal, id, sizeof(u.internal));
    const nccl_result r = a.comm_init_rank(&t->comm, world, u, rank);
    if (r != 0) {
        delete t;
        return set_error(KGS_ENCCL, std::string("ncclCommInitRank: ") + a.error_string(r));
    }
    out->ctx = t;
    out->all_gather = nccl_all_gather;
    out->all_reduce_sum_i64 = nccl_all_reduce_i64;
    out->owned = 1;
    return KGS_OK;
}

void kgs_vp_transport_free(kgs_vp_transport *t) {
    if (!t || !t->owned || !t->ctx) return;
    auto *x = static_cast<NcclTransport *>(t->ctx);
    if (x->comm) x->api.comm_destroy(x->comm);
    delete x;
    t->ctx = nullptr;
    t->owned = 0;
}

kgs_status kgs_vp_query(kgs_graph *g, const int32_t *kw_ids, int32_t q, int32_t k, const kgs_params *pp, int32_t rank,
                        int32_t world, const kgs_vp_transport *t, void *cuda_stream, kgs_result **out) {
    if (!g || !kw_ids || !out || !t || !t->all_gather || !t->all_reduce_sum_i64)
        return set_error(KGS_EINVAL, "null argument / incomplete transport");
    if (world < 1 || rank < 0 || rank >= world) return set_error(KGS_EINVAL, "rank / world out of range");
    *out = nullptr;
    kgs_params p;
    if (pp) p = *pp; else kgs_params_default(&p);
    cudaStream_t s = (cudaStream_t)cuda_stream;
    kgs_status st = KGS_OK;
    const int64_t n = graph_nodes(g);
    const int64_t slice = kgs_vp_slice(n, world), n_pad = slice * world;
    uint8_t *hm = nullptr, *hm_slice = nullptr, *M = nullptr, *Mown = nullptr, *cdep = nullptr, *dall = nullptr;
    int64_t *counts = nullptr, *mychg = nullptr, *allchg = nullptr, *cn = nullptr, *cnall = nullptr;
    int32_t *cent = nullptr, *cent_n = nullptr, *call = nullptr, *cfin = nullptr;
    long long *chg = nullptr, *chgpad = nullptr, *chgall = nullptr;
    uint8_t *dfin = nullptr;
    int64_t h_counts[4] = {0, 0, 0, 0};
    int32_t info[2] = {0, 0};
    int level = 0, stop = KGS_STOP_EXHAUSTED;
    int64_t n_central = 0;
    std::vector<int64_t> per(world);
    Coll coll{t, world, s, {}, {}};
    VQ_TRY(cudaSetDevice(graph_device(g)));
    VQ_TRY(cudaMallocAsync((void **)&hm, (size_t)n_pad, s));
    VQ_TRY(cudaMallocAsync((void **)&hm_slice, (size_t)std::max<int64_t>(slice, 1), s));
    VQ_TRY(cudaMallocAsync((void **)&M, (size_t)n_pad * 8, s));
    VQ_TRY(cudaMallocAsync((void **)&Mown, (size_t)std::max<int64_t>(slice, 1) * 8, s));
    VQ_TRY(cudaMallocAsync((void **)&counts, 4 * sizeof(int64_t), s));
    VQ_TRY(cudaMallocAsync((void **)&mychg, sizeof(int64_t), s));
    VQ_TRY(cudaMallocAsync((void **)&allchg, sizeof(int64_t) * world, s));
    VQ_TRY(cudaMallocAsync((void **)&cent, sizeof(int32_t) * std::max<int64_t>(slice, 1), s));
    VQ_TRY(cudaMallocAsync((void **)&cdep, (size_t)std::max<int64_t>(slice, 1), s));
    VQ_TRY(cudaMallocAsync((void **)&cent_n, sizeof(int32_t), s));
    VQ_TRY(cudaMallocAsync((void **)&chg, sizeof(long long) * std::max<int64_t>(slice, 1), s));
    VQ_TRY(cudaMemsetAsync(M, 0xFF, (size_t)n_pad * 8, s));
    VQ_TRY(cudaMemsetAsync(hm_slice, 0, (size_t)std::max<int64_t>(slice, 1), s));
    {
        kgs_vp_buffers b{};
        b.hm = hm; b.hm_slice = hm_slice; b.M = M; b.counts = counts; b.cent = cent; b.cdep = cdep;
        b.cent_n = cent_n; b.chg = reinterpret_cast<int64_t *>(chg);
        VQ_OK(kgs_vp_begin(g, kw_ids, q, k, &p, rank, world, &b, cuda_stream, info));
    }
    if (info[1]) {   // reading R17: some T_i is empty, nothing can be central
        stop = KGS_STOP_EMPTY_KEYWORD;
        level = 0;
    } else {
        VQ_COLL(coll.all_reduce_i64(counts, 4));
        VQ_TRY(cudaMemcpyAsync(h_counts, counts, sizeof(h_counts), cudaMemcpyDeviceToHost, s));
        VQ_TRY(cudaStreamSynchronize(s));
        n_central = h_counts[1];
        const int amax = info[0];
        for (;;) {
            if (n_central >= k) { stop = KGS_STOP_K; break; }               // Def. 4 / Thm. V.3 (R9)
            if (level == p.max_depth) { stop = KGS_STOP_MAX_DEPTH; break; }
            VQ_OK(kgs_vp_level(g, level, cuda_stream));
            VQ_TRY(cudaMemcpyAsync(mychg, counts + 3, sizeof(int64_t), cudaMemcpyDeviceToDevice, s));
            VQ_COLL(coll.all_reduce_i64(counts, 4));
            VQ_TRY(cudaMemcpyAsync(h_counts, counts, sizeof(h_counts), cudaMemcpyDeviceToHost, s));
            VQ_TRY(cudaStreamSynchronize(s));
            // exchange of the owned hit masks: sparse when few nodes changed in total, dense otherwise
            if (h_counts[3] * 16 < n) {
                VQ_COLL(coll.all_gather(mychg, allchg, sizeof(int64_t)));
                VQ_TRY(cudaMemcpyAsync(per.data(), allchg, sizeof(int64_t) * world, cudaMemcpyDeviceToHost, s));
                VQ_TRY(cudaStreamSynchronize(s));
                const int64_t width = std::max<int64_t>(1, *std::max_element(per.begin(), per.end()));
                VQ_TRY(cudaMallocAsync((void **)&chgpad, sizeof(long long) * width, s));
                VQ_TRY(cudaMallocAsync((void **)&chgall, sizeof(long long) * width * world, s));
                VQ_TRY(cudaMemsetAsync(chgpad, 0xFF, sizeof(long long) * width, s));
                if (per[rank]) VQ_TRY(cudaMemcpyAsync(chgpad, chg, sizeof(long long) * per[rank], cudaMemcpyDeviceToDevice, s));
                VQ_COLL(coll.all_gather(chgpad, chgall, (int64_t)sizeof(long long) * width));
                VQ_TRY(launch_vp_apply(chgall, width * world, hm, s));
                cudaFreeAsync(chgpad, s);
                cudaFreeAsync(chgall, s);
                chgpad = chgall = nullptr;
            } else {
                VQ_COLL(coll.all_gather(hm_slice, hm, slice));
            }
            const int64_t marks = h_counts[0];
            int64_t waiting = h_counts[2];
            n_central += h_counts[1];
            if (marks == 0 && waiting == 0 && level + 1 < amax) {   // a gated neighbour can still open (R22)
                VQ_OK(kgs_vp_waiting(g, level, cuda_stream));
                VQ_COLL(coll.all_reduce_i64(counts, 4));
                VQ_TRY(cudaMemcpyAsync(h_counts, counts, sizeof(h_counts), cudaMemcpyDeviceToHost, s));
                VQ_TRY(cudaStreamSynchronize(s));
                waiting = h_counts[2];
            }
            ++level;
            if (marks == 0 && waiting == 0) { stop = KGS_STOP_EXHAUSTED; break; }   // Alg. 2's list is empty
        }
        // the owned M rows and the central lists to every rank
        if (slice) VQ_TRY(cudaMemcpyAsync(Mown, M + (size_t)rank * slice * 8, (size_t)slice * 8, cudaMemcpyDeviceToDevice, s));
        VQ_COLL(coll.all_gather(Mown, M, slice * 8));
    }
    {
        int32_t my_n = 0;
        VQ_TRY(cudaMemcpyAsync(&my_n, cent_n, sizeof(int32_t), cudaMemcpyDeviceToHost, s));
        VQ_TRY(cudaStreamSynchronize(s));
        if (info[1]) my_n = 0;
        VQ_TRY(cudaMallocAsync((void **)&cn, sizeof(int64_t), s));
        VQ_TRY(cudaMallocAsync((void **)&cnall, sizeof(int64_t) * world, s));
        const int64_t my64 = my_n;
        VQ_TRY(cudaMemcpyAsync(cn, &my64, sizeof(int64_t), cudaMemcpyHostToDevice, s));
        VQ_COLL(coll.all_gather(cn, cnall, sizeof(int64_t)));
        VQ_TRY(cudaMemcpyAsync(per.data(), cnall, sizeof(int64_t) * world, cudaMemcpyDeviceToHost, s));
        VQ_TRY(cudaStreamSynchronize(s));
        const int64_t width = std::max<int64_t>(1, *std::max_element(per.begin(), per.end()));
        int64_t total = 0;
        for (int r = 0; r < world; ++r) total += per[r];
        int32_t *cpad = nullptr;
        uint8_t *dpad = nullptr;
        VQ_TRY(cudaMallocAsync((void **)&cpad, sizeof(int32_t) * width, s));
        VQ_TRY(cudaMallocAsync((void **)&dpad, (size_t)width, s));
        VQ_TRY(cudaMallocAsync((void **)&call, sizeof(int32_t) * width * world, s));
        VQ_TRY(cudaMallocAsync((void **)&dall, (size_t)width * world, s));
        VQ_TRY(cudaMallocAsync((void **)&cfin, sizeof(int32_t) * std::max<int64_t>(total, 1), s));
        VQ_TRY(cudaMallocAsync((void **)&dfin, (size_t)std::max<int64_t>(total, 1), s));
        if (my_n) {
            VQ_TRY(cudaMemcpyAsync(cpad, cent, sizeof(int32_t) * my_n, cudaMemcpyDeviceToDevice, s));
            VQ_TRY(cudaMemcpyAsync(dpad, cdep, (size_t)my_n, cudaMemcpyDeviceToDevice, s));
        }
        VQ_COLL(coll.all_gather(cpad, call, (int64_t)sizeof(int32_t) * width));
        VQ_COLL(coll.all_gather(dpad, dall, width));
        int64_t at = 0;   // rank blocks in rank order (the ranks' own identification order inside)
        for (int r = 0; r < world; ++r) {
            if (per[r]) {
                VQ_TRY(cudaMemcpyAsync(cfin + at, call + (size_t)r * width, sizeof(int32_t) * per[r], cudaMemcpyDeviceToDevice, s));
                VQ_TRY(cudaMemcpyAsync(dfin + at, dall + (size_t)r * width, (size_t)per[r], cudaMemcpyDeviceToDevice, s));
            }
            at += per[r];
        }
        cudaFreeAsync(cpad, s);
        cudaFreeAsync(dpad, s);
        if (!info[1] && total != n_central) {
            st = set_error(KGS_EINTERNAL, "vertex partition: gathered central lists disagree with the counters");
            goto done;
        }
        // the replicated final state (hm, M) is in the buffers kgs_vp_begin registered: the top-down reads them
        VQ_OK(kgs_vp_topdown(g, total, cfin, dfin, level, stop, cuda_stream, out));
    }
done:
    void *bufs[] = {hm, hm_slice, M, Mown, counts, mychg, allchg, cent, cdep, cent_n, chg, chgpad, chgall, cn, cnall,
                    call, dall, cfin, dfin};
    for (void *b : bufs) if (b) cudaFreeAsync(b, s);
    cudaStreamSynchronize(s);
    return st;
}

}  // extern "C"
