// ipt_api.cpp -- the C ABI of libipt (include/ipt.h): argument validation, plan
// execution (stage sequencing on one stream), workspace management, diagnostics.
//
// Stage sequence (Sec. 4.2) for `count` matrices at base + t*stride:
//   stage 1  100!  P(count, M, N', n)          -> cycle_global  (or identity)
//   stage 2  0010! P(count*N'*M', m, n, 1)     -> tile_onchip / cycle_global (or identity)
//   stage 3  0100! P(count*N', M', n, m)       -> cycle_global  (or identity)
// The batch is folded into every stage (the instances are independent), so each
// stage is a single launch regardless of `count`.
#include <nvtx3/nvToolsExt.h>
#include "ipt_internal.h"

#include <cstdio>

#include <algorithm>
#include <atomic>
#include <cstdlib>
#include <cstring>
#include <map>
#include <mutex>
#include <string>
#include <vector>

namespace ipt {

ipt_status plan_search(int64_t M, int64_t N, int eb, int device, ipt_plan_t *out);
std::vector<std::pair<int64_t, int64_t>> plan_candidates(int64_t M, int64_t N, int eb,
                                                         int device, int k);
void remember_tuned(int64_t M, int64_t N, int eb, int device, int64_t m, int64_t n);
void fill_plan(int64_t M, int64_t N, int64_t m, int64_t n, int eb, int device, ipt_plan_t *out);

static std::atomic<uint64_t> g_launches{0};
void note_launch() { g_launches.fetch_add(1, std::memory_order_relaxed); }

// Tuning knobs (IPT_* environment variables; tests and measurements only).  The launch
// path reads dozens of them per stage, so instead of a getenv (a scan of the whole
// environment) per read, the IPT_* entries are snapshot once per thread and re-scanned
// only when the environment block changes (environ pointer, entry count or the IPT_*
// strings -- what setenv/putenv, and so Python's os.environ, modify).
extern "C" char **environ;

namespace {
struct EnvSnap {
    char **env = nullptr;
    size_t count = 0;
    uint64_t hash = 0;
    std::vector<std::pair<std::string, std::string>> kv;
};
thread_local EnvSnap g_env;

void env_scan(EnvSnap &s) {
    s.env = environ;
    s.count = 0;
    s.kv.clear();
    uint64_t h = 1469598103934665603ull;
    for (char **e = environ; e && *e; ++e) {
        ++s.count;
        if (std::strncmp(*e, "IPT_", 4) != 0) continue;
        const char *eq = std::strchr(*e, '=');
        if (!eq) continue;
        s.kv.emplace_back(std::string(*e, eq - *e), std::string(eq + 1));
        for (const char *c = *e; *c; ++c) h = (h ^ (uint8_t)*c) * 1099511628211ull;
    }
    s.hash = h;
}

// Cheap check that the snapshot is current: same environ block and entry count, and each
// recorded IPT_* value still the same (getenv only for the few IPT_* names present).
const EnvSnap &env_now() {
    EnvSnap &s = g_env;
    bool fresh = s.env == environ && s.env != nullptr;
    if (fresh) {
        size_t n = 0;
        for (char **e = environ; *e; ++e) ++n;
        fresh = n == s.count;
        for (size_t i = 0; fresh && i < s.kv.size(); ++i) {
            const char *v = std::getenv(s.kv[i].first.c_str());
            fresh = v && s.kv[i].second == v;
        }
    }
    if (!fresh) env_scan(s);
    return s;
}
}  // namespace

long env_int(const char *name, long dflt) {
    const EnvSnap &s = env_now();
    for (const auto &kv : s.kv) {
        if (kv.first != name) continue;
        const char *v = kv.second.c_str();
        if (!*v) return dflt;
        char *end = nullptr;
        long x = std::strtol(v, &end, 10);
        return (end && *end == 0) ? x : dflt;
    }
    return dflt;
}

uint64_t env_hash() { return env_now().hash; }

FastDiv make_fastdiv(uint64_t d) {
    FastDiv f{};
    if (d == 0) d = 1;
    f.d = d;
    uint32_t l = 0;
    if (d > 1) l = 64 - (uint32_t)__builtin_clzll(d - 1);   // ceil(log2 d)
    unsigned __int128 two_l = (unsigned __int128)1 << l;
    unsigned __int128 m = ((two_l - d) << 64) / d + 1;
    f.m = (uint64_t)m;
    f.s1 = l ? 1 : 0;
    f.s2 = l ? l - 1 : 0;
    return f;
}

FastDiv32 make_fastdiv32(uint32_t d) {
    FastDiv32 f{};
    if (d == 0) d = 1;
    f.d = d;
    uint32_t l = 0;
    if (d > 1) l = 32 - (uint32_t)__builtin_clz(d - 1);
    const uint64_t two_l = (uint64_t)1 << l;
    f.m = (uint32_t)((((two_l - d) << 32) / d) + 1);
    f.s1 = l ? 1 : 0;
    f.s2 = l ? l - 1 : 0;
    return f;
}

DevProps dev_props(int device) {
    static std::mutex mu;
    static std::map<int, DevProps> cache;
    std::lock_guard<std::mutex> lk(mu);
    auto it = cache.find(device);
    if (it != cache.end()) return it->second;
    DevProps p{};
    // nominal B200 (sm_100a) values, used when planning without a device (device < 0)
    p.sms = 148;
    p.smem_optin = 232448;
    p.smem_per_sm = 233472;
    p.max_threads_sm = 2048;
    p.l2_bytes = 126 * 1024 * 1024;
    p.valid = device < 0;
    if (device >= 0) {
        int v = 0;
        if (cudaDeviceGetAttribute(&v, cudaDevAttrMultiProcessorCount, device) == cudaSuccess) {
            p.sms = v;
            p.valid = true;
            cudaDeviceGetAttribute(&p.smem_optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, device);
            cudaDeviceGetAttribute(&p.smem_per_sm, cudaDevAttrMaxSharedMemoryPerMultiprocessor, device);
            cudaDeviceGetAttribute(&p.max_threads_sm, cudaDevAttrMaxThreadsPerMultiProcessor, device);
            cudaDeviceGetAttribute(&p.l2_bytes, cudaDevAttrL2CacheSize, device);
        } else {
            cudaGetLastError();
        }
    }
    cache[device] = p;
    return p;
}

}  // namespace ipt

using namespace ipt;

namespace {

bool elem_ok(int eb) { return eb == 1 || eb == 2 || eb == 4 || eb == 8 || eb == 16; }

bool mul_ok(int64_t a, int64_t b, int64_t *out) {
    if (a < 0 || b < 0) return false;
    if (a == 0 || b == 0) { *out = 0; return true; }
    if (a > INT64_MAX / b) return false;
    *out = a * b;
    return true;
}

ipt_status check_shape(int64_t M, int64_t N, int eb, int64_t *bytes) {
    if (!elem_ok(eb)) return IPT_ERR_UNSUPPORTED_ELEM;
    if (M < 1 || N < 1) return IPT_ERR_INVALID_ARG;
    int64_t mn = 0, b = 0;
    if (!mul_ok(M, N, &mn) || !mul_ok(mn, eb, &b)) return IPT_ERR_INVALID_ARG;
    if (bytes) *bytes = b;
    return IPT_OK;
}

int current_device() {
    int d = 0;
    if (cudaGetDevice(&d) != cudaSuccess) {
        cudaGetLastError();
        return -1;
    }
    return d;
}

// Internal workspace cache, one buffer per (device, stream).
struct WsCache {
    std::mutex mu;
    std::map<std::pair<int, void *>, std::pair<void *, size_t>> bufs;
};
WsCache &ws_cache() {
    static WsCache *c = new WsCache();   // leaked on purpose: outlives CUDA teardown
    return *c;
}

// Internal buffers are cached per (device, stream, purpose): `purpose` 0 = flag workspace,
// 1 = host-path staging buffer, 2 = host pipeline buffers.  A flag workspace that must grow
// is RETIRED, not freed: work already enqueued on the stream -- or a CUDA graph captured
// from it by the caller -- may still hold the old pointer, so it stays valid until process
// exit (flag workspaces are small: one bit per unit).  Staging buffers (whole
// matrices) are freed after synchronising the stream; the host paths refuse stream capture.
bool stream_capturing(cudaStream_t st) {
    cudaStreamCaptureStatus cap = cudaStreamCaptureStatusNone;
    if (cudaStreamIsCapturing(st, &cap) != cudaSuccess) {
        cudaGetLastError();
        return true;   // unknown: treat as capturing (no synchronising calls)
    }
    return cap != cudaStreamCaptureStatusNone;
}

ipt_status get_ws(int device, void *stream, size_t need, void **out, int purpose = 0) {
    if (need == 0) { *out = nullptr; return IPT_OK; }
    WsCache &c = ws_cache();
    std::lock_guard<std::mutex> lk(c.mu);
    auto key = std::make_pair(device * 4 + purpose, stream);
    auto it = c.bufs.find(key);
    if (it != c.bufs.end() && it->second.second >= need) {
        *out = it->second.first;
        return IPT_OK;
    }
    if (it != c.bufs.end()) {
        if (purpose != 0) {
            if (stream_capturing((cudaStream_t)stream)) return IPT_ERR_INVALID_ARG;
            cudaStreamSynchronize((cudaStream_t)stream);
            cudaFree(it->second.first);
        }   // purpose 0: retired, never freed (see above)
        c.bufs.erase(it);
    }
    size_t sz = need < (1u << 20) ? (1u << 20) : need + need / 4;
    void *p = nullptr;
    if (cudaMalloc(&p, sz) != cudaSuccess) {
        cudaGetLastError();
        return IPT_ERR_NO_MEMORY;
    }
    c.bufs[key] = std::make_pair(p, sz);
    *out = p;
    return IPT_OK;
}

// Flag workspace of one call: the caller's (checked), else a graph-owned allocation under
// stream capture (released by release_ws at the end of the captured sequence), else the
// per-stream cache.
struct CallWs {
    void *ptr = nullptr;
    bool graph_owned = false;
};

ipt_status acquire_ws(int device, cudaStream_t st, size_t need, void *user, size_t user_bytes, CallWs *w) {
    w->graph_owned = false;
    if (user) {
        if (user_bytes < need) return IPT_ERR_NO_MEMORY;
        w->ptr = user;
        return IPT_OK;
    }
    if (need && stream_capturing(st)) {
        if (cudaMallocAsync(&w->ptr, need, st) != cudaSuccess) {
            cudaGetLastError();
            return IPT_ERR_NO_MEMORY;
        }
        w->graph_owned = true;
        return IPT_OK;
    }
    return get_ws(device, (void *)st, need, &w->ptr);
}

cudaError_t release_ws(const CallWs &w, cudaStream_t st, cudaError_t e) {
    if (!w.graph_owned) return e;
    const cudaError_t f = cudaFreeAsync(w.ptr, st);
    return e != cudaSuccess ? e : f;
}

thread_local cudaError_t g_last_cuda = cudaSuccess;

ipt_status cuda_status(cudaError_t e) {
    if (e == cudaSuccess) return IPT_OK;
    g_last_cuda = e;
    cudaGetLastError();
    return IPT_ERR_CUDA;
}

void rec(void *const *events, int i, cudaStream_t st) {
    if (events && events[i]) cudaEventRecord((cudaEvent_t)events[i], st);
}

// Stage descriptors of a plan applied to `count` matrices.
void plan_stages(const ipt_plan_t *p, char *base, int64_t count, int64_t stride, StageDesc st[3]) {
    for (int i = 0; i < 3; ++i) {
        st[i] = StageDesc{};
        st[i].base = base;
        st[i].outer = count;
        st[i].ostride = stride;
        st[i].eb = p->elem_bytes;
    }
    st[0].inner = 1;            st[0].A = p->M;  st[0].B = p->Np; st[0].s = p->n;
    st[1].inner = p->Np * p->Mp; st[1].A = p->m;  st[1].B = p->n;  st[1].s = 1;
    st[2].inner = p->Np;        st[2].A = p->Mp; st[2].B = p->n;  st[2].s = p->m;
}

ipt_status validate_plan(const ipt_plan_t *p) {
    if (!p) return IPT_ERR_INVALID_ARG;
    ipt_status s = check_shape(p->M, p->N, p->elem_bytes, nullptr);
    if (s) return s;
    if (p->m < 1 || p->n < 1 || p->M % p->m || p->N % p->n || p->Mp != p->M / p->m ||
        p->Np != p->N / p->n)
        return IPT_ERR_INVALID_ARG;
    // Stage 1 P(1, M, N', n) and stage 3 P(N', M', n, m) move super-elements by cycle
    // following; stage 2 P(N'M', m, n, 1) is tile-local (on chip, square swap, or cycle
    // following when the tile does not fit).  A stage may be the identity only when one of
    // its swapped dimensions is 1 -- a plan edited otherwise is rejected.
    const int *v = p->variant;
    const bool id1 = p->M == 1 || p->Np == 1, id2 = p->m == 1 || p->n == 1, id3 = p->Mp == 1 || p->n == 1;
    if (!(v[0] == IPT_VAR_CYCLE_GLOBAL || (v[0] == IPT_VAR_IDENTITY && id1))) return IPT_ERR_INVALID_ARG;
    if (!(v[2] == IPT_VAR_CYCLE_GLOBAL || (v[2] == IPT_VAR_IDENTITY && id3))) return IPT_ERR_INVALID_ARG;
    if (!(v[1] == IPT_VAR_CYCLE_GLOBAL || v[1] == IPT_VAR_TILE_ONCHIP ||
          (v[1] == IPT_VAR_SQUARE_SWAP && p->m == p->n) || (v[1] == IPT_VAR_IDENTITY && id2)))
        return IPT_ERR_INVALID_ARG;
    return IPT_OK;
}

size_t batched_ws(const ipt_plan_t *p, int64_t count) {
    StageDesc st[3];
    plan_stages(p, nullptr, count, p->M * p->N * p->elem_bytes, st);
    size_t ws = 0;
    for (int i = 0; i < 3; ++i) {
        if (p->variant[i] == IPT_VAR_CYCLE_GLOBAL) ws = std::max(ws, cycle_ws_bytes(st[i]));
        if (p->variant[i] == IPT_VAR_TILE_ONCHIP) ws = std::max(ws, kTileWsBytes);
    }
    return ws;
}

ipt_status run_plan(char *base, int64_t count, int64_t stride, const ipt_plan_t *p, void *ws,
                    size_t ws_bytes, cudaStream_t st, void *const *events) {
    const int device = current_device();
    if (device < 0) return IPT_ERR_NO_DEVICE;
    const size_t need = batched_ws(p, count);
    // Under stream capture (e.g. torch.cuda.graph) without a caller workspace, the flags
    // live in a graph-owned allocation (cudaMallocAsync / cudaFreeAsync nodes): every
    // replay gets its own workspace, so replays on other streams never share flags or
    // counters with direct calls on the capture stream.
    CallWs w;
    if (ipt_status s = acquire_ws(device, st, need, ws, ws_bytes, &w)) return s;
    ws = w.ptr;
    StageDesc sd[3];
    plan_stages(p, base, count, stride, sd);
    rec(events, 0, st);
    cudaError_t e = cudaSuccess;
    // NVTX range per launched stage (header-only NVTX3: a no-op unless a profiler injects
    // itself): nsys/ncu timelines and `ncu --nvtx --nvtx-include "ipt 0010!/"` filters
    static const char *const kStageNames[3] = {"ipt 100! (stage 1)", "ipt 0010! (stage 2)",
                                               "ipt 0100! (stage 3)"};
    const bool nvtx = env_int("IPT_NVTX", 1) != 0;
    for (int i = 0; i < 3 && e == cudaSuccess; ++i) {
        const bool ranged = nvtx && p->variant[i] != IPT_VAR_IDENTITY;
        if (ranged) nvtxRangePushA(kStageNames[i]);
        switch (p->variant[i]) {
            case IPT_VAR_IDENTITY: break;
            case IPT_VAR_TILE_ONCHIP: e = launch_tile_onchip(sd[i], ws, st, device); break;
            case IPT_VAR_SQUARE_SWAP: e = launch_square_swap(sd[i], st, device); break;
            case IPT_VAR_CYCLE_GLOBAL: e = launch_cycle_global(sd[i], ws, st, device); break;
            default: e = cudaErrorInvalidValue; break;
        }
        if (ranged) nvtxRangePop();
        if (e == cudaSuccess) rec(events, i + 1, st);
    }
    return cuda_status(release_ws(w, st, e));
}

ipt_status check_ptr(const void *p, int eb) {
    if (!p) return IPT_ERR_INVALID_ARG;
    if (((uintptr_t)p) % (uintptr_t)eb) return IPT_ERR_MISALIGNED;
    return IPT_OK;
}

}  // namespace

extern "C" {

ipt_status ipt_plan(int64_t M, int64_t N, int elem_bytes, int device, ipt_plan_t *out) {
    if (!out) return IPT_ERR_INVALID_ARG;
    ipt_status s = check_shape(M, N, elem_bytes, nullptr);
    if (s) return s;
    return plan_search(M, N, elem_bytes, device, out);
}

ipt_status ipt_plan_with_tiles(int64_t M, int64_t N, int64_t m, int64_t n, int elem_bytes,
                               int device, ipt_plan_t *out) {
    if (!out) return IPT_ERR_INVALID_ARG;
    ipt_status s = check_shape(M, N, elem_bytes, nullptr);
    if (s) return s;
    if (m < 1 || n < 1 || M % m || N % n) return IPT_ERR_INVALID_ARG;
    fill_plan(M, N, m, n, elem_bytes, device, out);
    return IPT_OK;
}

size_t ipt_workspace_bytes(const ipt_plan_t *plan, int64_t batch) {
    if (validate_plan(plan) || batch < 0) return 0;
    return batched_ws(plan, batch);
}

ipt_status ipt_transpose_plan_events(void *d_ptr, const ipt_plan_t *plan, void *d_workspace,
                                     size_t ws_bytes, void *stream, void *const *events) {
    ipt_status s = validate_plan(plan);
    if (s) return s;
    if ((s = check_ptr(d_ptr, plan->elem_bytes))) return s;
    return run_plan((char *)d_ptr, 1, plan->M * plan->N * plan->elem_bytes, plan, d_workspace,
                    ws_bytes, (cudaStream_t)stream, events);
}

ipt_status ipt_transpose_plan(void *d_ptr, const ipt_plan_t *plan, void *d_workspace,
                              size_t ws_bytes, void *stream) {
    return ipt_transpose_plan_events(d_ptr, plan, d_workspace, ws_bytes, stream, nullptr);
}

ipt_status ipt_transpose(void *d_ptr, int64_t M, int64_t N, int elem_bytes, void *stream) {
    ipt_status s = check_shape(M, N, elem_bytes, nullptr);
    if (s) return s;
    if ((s = check_ptr(d_ptr, elem_bytes))) return s;
    if (M == 1 || N == 1) return IPT_OK;
    const int device = current_device();
    if (device < 0) return IPT_ERR_NO_DEVICE;
    ipt_plan_t p;
    if ((s = ipt_plan(M, N, elem_bytes, device, &p))) return s;
    return run_plan((char *)d_ptr, 1, M * N * elem_bytes, &p, nullptr, 0, (cudaStream_t)stream,
                    nullptr);
}

ipt_status ipt_transpose_batched_plan_events(void *d_base, int64_t count, int64_t stride_bytes,
                                             const ipt_plan_t *plan, void *d_workspace,
                                             size_t ws_bytes, void *stream,
                                             void *const *events) {
    ipt_status s = validate_plan(plan);
    if (s) return s;
    if (count < 0) return IPT_ERR_INVALID_ARG;
    if (count == 0) return IPT_OK;
    if ((s = check_ptr(d_base, plan->elem_bytes))) return s;
    const int64_t mat = plan->M * plan->N * plan->elem_bytes;
    if (count > 1 && (stride_bytes < mat || stride_bytes % plan->elem_bytes)) return IPT_ERR_INVALID_ARG;
    if (count == 1) stride_bytes = mat;
    int64_t tot = 0;
    if (!mul_ok(count - 1, stride_bytes, &tot) || tot > INT64_MAX - mat) return IPT_ERR_INVALID_ARG;
    return run_plan((char *)d_base, count, stride_bytes, plan, d_workspace, ws_bytes,
                    (cudaStream_t)stream, events);
}

ipt_status ipt_transpose_batched_plan(void *d_base, int64_t count, int64_t stride_bytes,
                                      const ipt_plan_t *plan, void *d_workspace,
                                      size_t ws_bytes, void *stream) {
    return ipt_transpose_batched_plan_events(d_base, count, stride_bytes, plan, d_workspace,
                                             ws_bytes, stream, nullptr);
}

ipt_status ipt_transpose_batched(void *d_base, int64_t count, int64_t stride_bytes, int64_t M,
                                 int64_t N, int elem_bytes, void *stream) {
    ipt_status s = check_shape(M, N, elem_bytes, nullptr);
    if (s) return s;
    if (count < 0) return IPT_ERR_INVALID_ARG;
    if (count == 0 || M == 1 || N == 1) return IPT_OK;
    if ((s = check_ptr(d_base, elem_bytes))) return s;
    const int64_t mat = M * N * elem_bytes;
    if (count > 1 && (stride_bytes < mat || stride_bytes % elem_bytes)) return IPT_ERR_INVALID_ARG;
    const int device = current_device();
    if (device < 0) return IPT_ERR_NO_DEVICE;
    ipt_plan_t p;
    if ((s = ipt_plan(M, N, elem_bytes, device, &p))) return s;
    return ipt_transpose_batched_plan(d_base, count, stride_bytes, &p, nullptr, 0, stream);
}

// ----------------------------------------------------------- elementary transpositions
static ipt_status check_stage(void *d, int64_t batch, int64_t A, int64_t B, int64_t s, int eb) {
    if (!elem_ok(eb)) return IPT_ERR_UNSUPPORTED_ELEM;
    if (batch < 0 || A < 1 || B < 1 || s < 1) return IPT_ERR_INVALID_ARG;
    int64_t x = 0;
    if (!mul_ok(batch, A, &x) || !mul_ok(x, B, &x) || !mul_ok(x, s, &x) || !mul_ok(x, eb, &x))
        return IPT_ERR_INVALID_ARG;
    if (batch == 0 || A == 1 || B == 1) return IPT_OK;
    return check_ptr(d, eb);
}

static StageDesc stage_desc(void *d, int64_t batch, int64_t A, int64_t B, int64_t s, int eb) {
    StageDesc sd{};
    sd.base = (char *)d;
    sd.outer = batch;
    sd.inner = 1;
    sd.ostride = A * B * s * eb;
    sd.A = A; sd.B = B; sd.s = s; sd.eb = eb;
    return sd;
}

size_t ipt_stage_workspace_bytes(int64_t batch, int64_t A, int64_t B, int64_t s, int elem_bytes) {
    if (check_stage((void *)16, batch, A, B, s, elem_bytes) != IPT_OK) return 0;
    if (batch == 0 || A == 1 || B == 1) return 0;
    const size_t c = cycle_ws_bytes(stage_desc(nullptr, batch, A, B, s, elem_bytes));
    return s == 1 ? std::max(c, kTileWsBytes) : c;
}

static ipt_status run_cycle(void *d, int64_t batch, int64_t A, int64_t B, int64_t s, int eb,
                            void *ws, size_t ws_bytes, void *stream) {
    ipt_status st = check_stage(d, batch, A, B, s, eb);
    if (st) return st;
    if (batch == 0 || A == 1 || B == 1) return IPT_OK;
    const int device = current_device();
    if (device < 0) return IPT_ERR_NO_DEVICE;
    StageDesc sd = stage_desc(d, batch, A, B, s, eb);
    CallWs w;
    if ((st = acquire_ws(device, (cudaStream_t)stream, cycle_ws_bytes(sd), ws, ws_bytes, &w))) return st;
    return cuda_status(release_ws(w, (cudaStream_t)stream,
                                  launch_cycle_global(sd, w.ptr, (cudaStream_t)stream, device)));
}

ipt_status ipt_100(void *d_ptr, int64_t batch, int64_t A, int64_t B, int64_t s, int elem_bytes,
                   void *d_workspace, size_t ws_bytes, void *stream) {
    return run_cycle(d_ptr, batch, A, B, s, elem_bytes, d_workspace, ws_bytes, stream);
}

ipt_status ipt_010(void *d_ptr, int64_t batch, int64_t A, int64_t B, int elem_bytes,
                   void *d_workspace, size_t ws_bytes, void *stream) {
    ipt_status st = check_stage(d_ptr, batch, A, B, 1, elem_bytes);
    if (st) return st;
    if (batch == 0 || A == 1 || B == 1) return IPT_OK;
    const int device = current_device();
    if (device < 0) return IPT_ERR_NO_DEVICE;
    if (A == B && prefer_square_swap(batch, A, elem_bytes, device)) {   // P:45, no workspace
        StageDesc sd = stage_desc(d_ptr, batch, A, B, 1, elem_bytes);
        return cuda_status(launch_square_swap(sd, (cudaStream_t)stream, device));
    }
    if (tile_onchip_fits(A, B, elem_bytes, device)) {
        StageDesc sd = stage_desc(d_ptr, batch, A, B, 1, elem_bytes);
        CallWs w;
        if ((st = acquire_ws(device, (cudaStream_t)stream, kTileWsBytes, d_workspace, ws_bytes, &w))) return st;
        return cuda_status(release_ws(w, (cudaStream_t)stream,
                                      launch_tile_onchip(sd, w.ptr, (cudaStream_t)stream, device)));
    }
    return run_cycle(d_ptr, batch, A, B, 1, elem_bytes, d_workspace, ws_bytes, stream);
}

ipt_status ipt_0010(void *d_ptr, int64_t d0, int64_t d1, int64_t d2, int64_t d3, int elem_bytes,
                    void *d_workspace, size_t ws_bytes, void *stream) {
    int64_t b = 0;
    if (d0 < 0 || d1 < 0 || !mul_ok(d0, d1, &b)) return IPT_ERR_INVALID_ARG;
    return ipt_010(d_ptr, b, d2, d3, elem_bytes, d_workspace, ws_bytes, stream);
}

ipt_status ipt_0100(void *d_ptr, int64_t d0, int64_t d1, int64_t d2, int64_t d3, int elem_bytes,
                    void *d_workspace, size_t ws_bytes, void *stream) {
    return ipt_100(d_ptr, d0, d1, d2, d3, elem_bytes, d_workspace, ws_bytes, stream);
}

ipt_status ipt_1000(void *d_ptr, int64_t d0, int64_t d1, int64_t d2, int64_t d3, int elem_bytes,
                    void *d_workspace, size_t ws_bytes, void *stream) {
    int64_t s = 0;
    if (d2 < 1 || d3 < 1 || !mul_ok(d2, d3, &s)) return IPT_ERR_INVALID_ARG;
    return ipt_100(d_ptr, 1, d0, d1, s, elem_bytes, d_workspace, ws_bytes, stream);
}

// ------------------------------------------------------------- measured plan choice
// Sec. 7.4 says exhaustive search is too slow and prunes it; here the cost model prunes
// to a few candidates and the device decides: each candidate transposes the caller's
// matrix (M x N -> N x M) and the model-best N x M plan transposes it back, so the data
// is unchanged on return.  The winner is remembered for (M, N, elem_bytes, device) and
// returned by ipt_plan / used by ipt_transpose from then on.
static ipt_status autotune_impl(void *d_ptr, int64_t count, int64_t stride, int64_t M,
                                int64_t N, int elem_bytes, int candidates, void *stream,
                                ipt_plan_t *out) {
    if (!out || count < 1) return IPT_ERR_INVALID_ARG;
    ipt_status s = check_shape(M, N, elem_bytes, nullptr);
    if (s) return s;
    if ((s = check_ptr(d_ptr, elem_bytes))) return s;
    const int64_t mat = M * N * elem_bytes;
    if (count == 1) stride = mat;
    if (count > 1 && (stride < mat || stride % elem_bytes)) return IPT_ERR_INVALID_ARG;
    const int device = current_device();
    if (device < 0) return IPT_ERR_NO_DEVICE;
    if (M == 1 || N == 1 || candidates < 2) return ipt_plan(M, N, elem_bytes, device, out);
    // Small jobs are latency-bound, where the cost model is least accurate and timing a
    // candidate costs microseconds: time at least 12.  Jobs that fit in L2 are timed cold
    // (an L2-sized scratch buffer is overwritten before every repetition, outside the
    // events), as a single call on fresh data would run.
    const int64_t job = mat + (count - 1) * stride;
    if (job <= ((int64_t)256 << 20) && candidates < 12) candidates = 12;
    void *flush = nullptr;
    size_t flush_bytes = 0;
    if (job < (int64_t)dev_props(device).l2_bytes) {
        static std::mutex fmu;
        static std::map<int, std::pair<void *, size_t>> fcache;
        std::lock_guard<std::mutex> lk(fmu);
        auto &f = fcache[device];
        if (!f.first) {
            f.second = (size_t)dev_props(device).l2_bytes * 2;
            if (cudaMalloc(&f.first, f.second) != cudaSuccess) { cudaGetLastError(); f.first = nullptr; }
        }
        flush = f.first;
        flush_bytes = f.second;
    }
    auto cands = plan_candidates(M, N, elem_bytes, device, candidates);
    ipt_plan_t back;
    if ((s = plan_search(N, M, elem_bytes, device, &back))) return s;
    cudaStream_t st = (cudaStream_t)stream;
    cudaEvent_t e0, e1;
    if (cudaEventCreate(&e0) != cudaSuccess || cudaEventCreate(&e1) != cudaSuccess)
        return cuda_status(cudaGetLastError());
    float best_ms = 0;
    int64_t bm = cands[0].first, bn = cands[0].second;
    for (size_t i = 0; i < cands.size(); ++i) {
        ipt_plan_t p;
        fill_plan(M, N, cands[i].first, cands[i].second, elem_bytes, device, &p);
        float t_min = 0;
        for (int rep = 0; rep < 2; ++rep) {
            if (flush) cudaMemsetAsync(flush, rep, flush_bytes, st);
            cudaEventRecord(e0, st);
            if ((s = run_plan((char *)d_ptr, count, stride, &p, nullptr, 0, st, nullptr))) break;
            cudaEventRecord(e1, st);
            if ((s = run_plan((char *)d_ptr, count, stride, &back, nullptr, 0, st, nullptr))) break;
            if (cudaEventSynchronize(e1) != cudaSuccess) { s = IPT_ERR_CUDA; break; }
            float ms = 0;
            cudaEventElapsedTime(&ms, e0, e1);
            if (rep == 0 || ms < t_min) t_min = ms;
        }
        if (s) break;
        if (env_int("IPT_DEBUG", 0))
            fprintf(stderr, "[ipt] autotune %lldx%lld cand m=%lld n=%lld var=%d,%d,%d ms=%.4f\n",
                    (long long)M, (long long)N, (long long)p.m, (long long)p.n, p.variant[0],
                    p.variant[1], p.variant[2], t_min);
        if (i == 0 || t_min < best_ms) { best_ms = t_min; bm = cands[i].first; bn = cands[i].second; }
    }
    cudaEventDestroy(e0);
    cudaEventDestroy(e1);
    if (s) return s;
    if (count == 1) remember_tuned(M, N, elem_bytes, device, bm, bn);
    fill_plan(M, N, bm, bn, elem_bytes, device, out);
    return IPT_OK;
}

ipt_status ipt_plan_autotune(void *d_ptr, int64_t M, int64_t N, int elem_bytes, int candidates,
                             void *stream, ipt_plan_t *out) {
    return autotune_impl(d_ptr, 1, 0, M, N, elem_bytes, candidates, stream, out);
}

ipt_status ipt_plan_autotune_batched(void *d_base, int64_t count, int64_t stride_bytes,
                                     int64_t M, int64_t N, int elem_bytes, int candidates,
                                     void *stream, ipt_plan_t *out) {
    return autotune_impl(d_base, count, stride_bytes, M, N, elem_bytes, candidates, stream, out);
}

// ---------------------------------------------- 4-stage baseline (Fig. 2; NEXT-2)
// Gustavson/Karlsson 4-stage sequence on the 4-D view M' x m x N' x n:
//   0100!  P(M', m, N', n)     M' instances of m x N' with n-element super-elements
//   0010!  P(M'N', m, n, 1)    every m x n tile
//   1000!  P(1, M', N', m*n)   one M' x N' array of (m*n)-element super-elements
//   0100!  P(N', M', n, m)     N' instances of M' x n with m-element super-elements
// Same kernels as the 3-stage path; kept as the paper's baseline for its 3x claim (Table 2).
ipt_status ipt_transpose_4stage(void *d_ptr, int64_t M, int64_t N, int64_t m, int64_t n,
                                int elem_bytes, void *d_workspace, size_t ws_bytes,
                                void *stream) {
    ipt_status s = check_shape(M, N, elem_bytes, nullptr);
    if (s) return s;
    if ((s = check_ptr(d_ptr, elem_bytes))) return s;
    if (m < 0 || n < 0 || (m && M % m) || (n && N % n)) return IPT_ERR_INVALID_ARG;
    if (M == 1 || N == 1) return IPT_OK;
    const int device = current_device();
    if (device < 0) return IPT_ERR_NO_DEVICE;
    if (!m || !n) {
        ipt_plan_t p;
        if ((s = ipt_plan(M, N, elem_bytes, device, &p))) return s;
        if (!m) m = p.m;
        if (!n) n = p.n;
    }
    const int64_t Mp = M / m, Np = N / n;
    StageDesc sd[4];
    for (int i = 0; i < 4; ++i) {
        sd[i] = StageDesc{};
        sd[i].base = (char *)d_ptr;
        sd[i].inner = 1;
        sd[i].eb = elem_bytes;
    }
    sd[0].outer = Mp;      sd[0].A = m;  sd[0].B = Np; sd[0].s = n;
    sd[1].outer = Mp * Np; sd[1].A = m;  sd[1].B = n;  sd[1].s = 1;
    sd[2].outer = 1;       sd[2].A = Mp; sd[2].B = Np; sd[2].s = m * n;
    sd[3].outer = Np;      sd[3].A = Mp; sd[3].B = n;  sd[3].s = m;
    size_t need = 0;
    bool tile2 = false, sq2 = false;
    for (int i = 0; i < 4; ++i) {
        sd[i].ostride = sd[i].A * sd[i].B * sd[i].s * elem_bytes;
        if (sd[i].A == 1 || sd[i].B == 1) continue;
        if (i == 1 && m == n && prefer_square_swap(Mp * Np, m, elem_bytes, device)) {
            sq2 = true;
            continue;
        }
        if (i == 1 && tile_onchip_fits(m, n, elem_bytes, device)) {
            tile2 = true;
            need = std::max(need, kTileWsBytes);
            continue;
        }
        need = std::max(need, cycle_ws_bytes(sd[i]));
    }
    CallWs w;
    if ((s = acquire_ws(device, (cudaStream_t)stream, need, d_workspace, ws_bytes, &w))) return s;
    void *ws = w.ptr;
    cudaError_t e = cudaSuccess;
    for (int i = 0; i < 4 && e == cudaSuccess; ++i) {
        if (sd[i].A == 1 || sd[i].B == 1) continue;
        e = (i == 1 && sq2)     ? launch_square_swap(sd[i], (cudaStream_t)stream, device)
            : (i == 1 && tile2) ? launch_tile_onchip(sd[i], ws, (cudaStream_t)stream, device)
                                : launch_cycle_global(sd[i], ws, (cudaStream_t)stream, device);
    }
    return cuda_status(release_ws(w, (cudaStream_t)stream, e));
}

// ------------------------------------------------- host-delegated transposition (Sec. 6)
// the matrix is copied to the GPU (1), transposed in place there (2), and
// copied back to the same host location (3).  Stage 1 (100!) spans the whole array and
// cannot be split; stages 2 and 3 work on independent instances, so the
// N' output panels are split into Q groups, each on its own stream: stage 2 + stage 3 +
// device-to-host copy of the group overlap with the other groups' work (Fig. 5b).
static ipt_status host_streams(int device, void *caller, int q, cudaStream_t *out) {
    // one set of Q streams per (device, caller stream): calls on different caller streams
    // never share queues, so asynchronous host calls on two streams overlap
    static std::mutex mu;
    static std::map<std::pair<int, void *>, std::vector<cudaStream_t>> cache;
    std::lock_guard<std::mutex> lk(mu);
    auto &v = cache[std::make_pair(device, caller)];
    while ((int)v.size() < q) {
        cudaStream_t s;
        if (cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking) != cudaSuccess) {
            cudaGetLastError();
            return IPT_ERR_CUDA;
        }
        v.push_back(s);
    }
    for (int i = 0; i < q; ++i) out[i] = v[i];
    return IPT_OK;
}

static size_t align256(size_t x) { return (x + 255) & ~(size_t)255; }

static ipt_status transpose_host_impl(void *h_ptr, int64_t M, int64_t N, int elem_bytes,
                                      int queues, void *d_buffer, size_t d_buffer_bytes,
                                      void *stream, bool sync) {
    int64_t bytes = 0;
    ipt_status s = check_shape(M, N, elem_bytes, &bytes);
    if (s) return s;
    if ((s = check_ptr(h_ptr, elem_bytes))) return s;
    if (queues < 1 || queues > 64) return IPT_ERR_INVALID_ARG;
    if (M == 1 || N == 1) return IPT_OK;
    const int device = current_device();
    if (device < 0) return IPT_ERR_NO_DEVICE;
    if (stream_capturing((cudaStream_t)stream)) return IPT_ERR_INVALID_ARG;
    ipt_plan_t p;
    if ((s = ipt_plan(M, N, elem_bytes, device, &p))) return s;
    const int64_t Np = p.Np;
    const int Q = (int)std::min<int64_t>(queues, Np);
    StageDesc sd[3];
    // workspace layout: [data | stage-1 flags | group 0 flags | group 1 flags | ...]
    plan_stages(&p, nullptr, 1, bytes, sd);
    size_t ws1 = p.variant[0] == IPT_VAR_CYCLE_GLOBAL ? cycle_ws_bytes(sd[0]) : 0;
    std::vector<int64_t> g0(Q + 1);
    for (int g = 0; g <= Q; ++g) g0[g] = Np * g / Q;
    std::vector<size_t> wsg(Q, 0);
    for (int g = 0; g < Q; ++g) {
        StageDesc a = sd[1], b = sd[2];
        a.inner = (g0[g + 1] - g0[g]) * p.Mp;
        b.inner = g0[g + 1] - g0[g];
        size_t w = 0;
        if (p.variant[1] == IPT_VAR_CYCLE_GLOBAL) w = std::max(w, cycle_ws_bytes(a));
        if (p.variant[1] == IPT_VAR_TILE_ONCHIP) w = std::max(w, kTileWsBytes);
        if (p.variant[2] == IPT_VAR_CYCLE_GLOBAL) w = std::max(w, cycle_ws_bytes(b));
        wsg[g] = align256(w);
    }
    size_t need = align256((size_t)bytes) + align256(ws1);
    for (size_t w : wsg) need += w;
    char *dbuf = (char *)d_buffer;
    cudaStream_t st = (cudaStream_t)stream;
    if (!dbuf) {
        void *w = nullptr;
        if ((s = get_ws(device, stream, need, &w, 1))) return s;
        dbuf = (char *)w;
    } else if (d_buffer_bytes < need) {
        return IPT_ERR_NO_MEMORY;
    }
    char *dws1 = dbuf + align256((size_t)bytes);
    std::vector<char *> dwsg(Q);
    char *cur = dws1 + align256(ws1);
    for (int g = 0; g < Q; ++g) { dwsg[g] = cur; cur += wsg[g]; }
    std::vector<cudaStream_t> qs(Q);
    if ((s = host_streams(device, stream, Q, qs.data()))) return s;

    cudaError_t e = cudaMemcpyAsync(dbuf, h_ptr, (size_t)bytes, cudaMemcpyHostToDevice, st);
    if (e != cudaSuccess) return cuda_status(e);
    plan_stages(&p, dbuf, 1, bytes, sd);
    if (p.variant[0] == IPT_VAR_CYCLE_GLOBAL) {
        if ((e = launch_cycle_global(sd[0], dws1, st, device)) != cudaSuccess) return cuda_status(e);
    }
    cudaEvent_t ev1;
    if ((e = cudaEventCreateWithFlags(&ev1, cudaEventDisableTiming)) != cudaSuccess) return cuda_status(e);
    cudaEventRecord(ev1, st);
    // panel q of the result (rows q*n .. q*n+n-1 of A^T) is the contiguous range
    // [q*M*n, (q+1)*M*n) elements, both after stage 1 (N' x M x n) and after stage 3.
    const int64_t panel = M * p.n * elem_bytes;
    std::vector<cudaEvent_t> done(Q);
    for (int g = 0; g < Q; ++g) {
        cudaStream_t qs_g = qs[g];
        cudaStreamWaitEvent(qs_g, ev1, 0);
        char *gb = dbuf + g0[g] * panel;
        const int64_t np_g = g0[g + 1] - g0[g];
        StageDesc a = sd[1], b = sd[2];
        a.base = gb; a.inner = np_g * p.Mp;
        b.base = gb; b.inner = np_g;
        if (p.variant[1] == IPT_VAR_TILE_ONCHIP) e = launch_tile_onchip(a, dwsg[g], qs_g, device);
        else if (p.variant[1] == IPT_VAR_SQUARE_SWAP) e = launch_square_swap(a, qs_g, device);
        else if (p.variant[1] == IPT_VAR_CYCLE_GLOBAL) e = launch_cycle_global(a, dwsg[g], qs_g, device);
        if (e != cudaSuccess) return cuda_status(e);
        if (p.variant[2] == IPT_VAR_CYCLE_GLOBAL) e = launch_cycle_global(b, dwsg[g], qs_g, device);
        if (e != cudaSuccess) return cuda_status(e);
        e = cudaMemcpyAsync((char *)h_ptr + g0[g] * panel, gb, (size_t)(np_g * panel),
                            cudaMemcpyDeviceToHost, qs_g);
        if (e != cudaSuccess) return cuda_status(e);
        cudaEventCreateWithFlags(&done[g], cudaEventDisableTiming);
        cudaEventRecord(done[g], qs_g);
        cudaStreamWaitEvent(st, done[g], 0);
    }
    e = sync ? cudaStreamSynchronize(st) : cudaGetLastError();
    cudaEventDestroy(ev1);   // released once the recorded work completes
    for (auto d : done) cudaEventDestroy(d);
    return cuda_status(e);
}

// Host pipeline (Sec. 6 across matrices): H2D of matrix i+1 and D2H of matrix i-1 overlap
// the stages of matrix i -- two device slots, a copy-in stream, a compute stream and a
// copy-out stream per (device, caller stream); slot reuse waits for its D2H.
static ipt_status pipe_streams(int device, void *caller, cudaStream_t out[3]) {
    static std::mutex mu;
    static std::map<std::pair<int, void *>, std::vector<cudaStream_t>> cache;
    std::lock_guard<std::mutex> lk(mu);
    auto &v = cache[std::make_pair(device, caller)];
    while (v.size() < 3) {
        cudaStream_t s;
        if (cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking) != cudaSuccess) {
            cudaGetLastError();
            return IPT_ERR_CUDA;
        }
        v.push_back(s);
    }
    for (int i = 0; i < 3; ++i) out[i] = v[i];
    return IPT_OK;
}

ipt_status ipt_transpose_host_pipeline(void *const *h_ptrs, const int64_t *Ms, const int64_t *Ns,
                                       int count, int elem_bytes, void *d_buffer,
                                       size_t d_buffer_bytes, void *stream) {
    if (count < 0 || (count > 0 && (!h_ptrs || !Ms || !Ns))) return IPT_ERR_INVALID_ARG;
    if (count == 0) return IPT_OK;
    if (!elem_ok(elem_bytes)) return IPT_ERR_UNSUPPORTED_ELEM;
    int64_t maxb = 0;
    for (int i = 0; i < count; ++i) {
        int64_t b = 0;
        ipt_status s = check_shape(Ms[i], Ns[i], elem_bytes, &b);
        if (s) return s;
        if ((s = check_ptr(h_ptrs[i], elem_bytes))) return s;
        maxb = std::max(maxb, b);
    }
    const int device = current_device();
    if (device < 0) return IPT_ERR_NO_DEVICE;
    if (stream_capturing((cudaStream_t)stream)) return IPT_ERR_INVALID_ARG;
    std::vector<ipt_plan_t> plans(count);
    size_t ws = 0;
    for (int i = 0; i < count; ++i) {
        if (Ms[i] == 1 || Ns[i] == 1) continue;
        ipt_status s = ipt_plan(Ms[i], Ns[i], elem_bytes, device, &plans[i]);
        if (s) return s;
        ws = std::max(ws, batched_ws(&plans[i], 1));
    }
    const size_t slot = align256((size_t)maxb);
    const size_t need = 2 * slot + align256(ws);
    char *dbuf = (char *)d_buffer;
    if (!dbuf) {
        void *w = nullptr;
        ipt_status s = get_ws(device, stream, need, &w, 2);
        if (s) return s;
        dbuf = (char *)w;
    } else if (d_buffer_bytes < need) {
        return IPT_ERR_NO_MEMORY;
    }
    char *dws = dbuf + 2 * slot;
    cudaStream_t qs[3];
    ipt_status s = pipe_streams(device, stream, qs);
    if (s) return s;
    cudaStream_t st = (cudaStream_t)stream, H = qs[0], C = qs[1], D = qs[2];
    cudaEvent_t start, h2d[2], comp[2], d2h[2];
    cudaEventCreateWithFlags(&start, cudaEventDisableTiming);
    for (int k = 0; k < 2; ++k) {
        cudaEventCreateWithFlags(&h2d[k], cudaEventDisableTiming);
        cudaEventCreateWithFlags(&comp[k], cudaEventDisableTiming);
        cudaEventCreateWithFlags(&d2h[k], cudaEventDisableTiming);
    }
    cudaEventRecord(start, st);               // everything follows prior work on `stream`
    cudaStreamWaitEvent(H, start, 0);
    cudaStreamWaitEvent(C, start, 0);
    cudaStreamWaitEvent(D, start, 0);
    cudaError_t e = cudaSuccess;
    for (int i = 0; i < count && e == cudaSuccess; ++i) {
        if (Ms[i] == 1 || Ns[i] == 1) continue;   // the layout is already its transpose
        const int k = i & 1;
        char *b = dbuf + k * slot;
        const size_t bytes = (size_t)(Ms[i] * Ns[i] * elem_bytes);
        if (i >= 2) cudaStreamWaitEvent(H, d2h[k], 0);   // slot k free again
        e = cudaMemcpyAsync(b, h_ptrs[i], bytes, cudaMemcpyHostToDevice, H);
        if (e != cudaSuccess) break;
        cudaEventRecord(h2d[k], H);
        cudaStreamWaitEvent(C, h2d[k], 0);
        ipt_status r = run_plan(b, 1, (int64_t)bytes, &plans[i], dws, align256(ws), C, nullptr);
        if (r) { e = cudaErrorUnknown; s = r; break; }
        cudaEventRecord(comp[k], C);
        cudaStreamWaitEvent(D, comp[k], 0);
        e = cudaMemcpyAsync(h_ptrs[i], b, bytes, cudaMemcpyDeviceToHost, D);
        if (e != cudaSuccess) break;
        cudaEventRecord(d2h[k], D);
    }
    // join: `stream` continues after every copy-out
    cudaEvent_t done;
    cudaEventCreateWithFlags(&done, cudaEventDisableTiming);
    cudaEventRecord(done, D);
    cudaStreamWaitEvent(st, done, 0);
    cudaEventRecord(done, C);                  // (re-recorded: C and H end before D anyway)
    cudaStreamWaitEvent(st, done, 0);
    cudaEventRecord(done, H);
    cudaStreamWaitEvent(st, done, 0);
    cudaEventDestroy(done);
    cudaEventDestroy(start);
    for (int k = 0; k < 2; ++k) {
        cudaEventDestroy(h2d[k]);
        cudaEventDestroy(comp[k]);
        cudaEventDestroy(d2h[k]);
    }
    if (s) return s;
    return cuda_status(e != cudaSuccess ? e : cudaGetLastError());
}

ipt_status ipt_transpose_host(void *h_ptr, int64_t M, int64_t N, int elem_bytes, int queues,
                              void *d_buffer, size_t d_buffer_bytes, void *stream) {
    return transpose_host_impl(h_ptr, M, N, elem_bytes, queues, d_buffer, d_buffer_bytes,
                               stream, true);
}

ipt_status ipt_transpose_host_async(void *h_ptr, int64_t M, int64_t N, int elem_bytes,
                                    int queues, void *d_buffer, size_t d_buffer_bytes,
                                    void *stream) {
    return transpose_host_impl(h_ptr, M, N, elem_bytes, queues, d_buffer, d_buffer_bytes,
                               stream, false);
}

// ------------------------------------------- layout marshaling (Sung's DL; NEXT-3)
// Array-of-Structures / Structure-of-Arrays <-> Array-of-Structures-of-Tiled-Arrays.
// AoS = M structures x N fields; ASTA groups the structures in tiles of m (M = M' m):
// M' x N x m.  AoS -> ASTA is 010! on M' x m x N; SoA (N x M' x m) -> ASTA is 100!
// (P:140).  The inverse transformations are the inverse elementary transpositions.
ipt_status ipt_aos_to_asta(void *d_ptr, int64_t M, int64_t N, int64_t m, int elem_bytes,
                           void *d_workspace, size_t ws_bytes, void *stream) {
    if (m < 1 || M < 1 || M % m) return IPT_ERR_INVALID_ARG;
    return ipt_010(d_ptr, M / m, m, N, elem_bytes, d_workspace, ws_bytes, stream);
}

ipt_status ipt_asta_to_aos(void *d_ptr, int64_t M, int64_t N, int64_t m, int elem_bytes,
                           void *d_workspace, size_t ws_bytes, void *stream) {
    if (m < 1 || M < 1 || M % m) return IPT_ERR_INVALID_ARG;
    return ipt_010(d_ptr, M / m, N, m, elem_bytes, d_workspace, ws_bytes, stream);
}

ipt_status ipt_soa_to_asta(void *d_ptr, int64_t M, int64_t N, int64_t m, int elem_bytes,
                           void *d_workspace, size_t ws_bytes, void *stream) {
    if (m < 1 || M < 1 || M % m) return IPT_ERR_INVALID_ARG;
    return ipt_100(d_ptr, 1, N, M / m, m, elem_bytes, d_workspace, ws_bytes, stream);
}

ipt_status ipt_asta_to_soa(void *d_ptr, int64_t M, int64_t N, int64_t m, int elem_bytes,
                           void *d_workspace, size_t ws_bytes, void *stream) {
    if (m < 1 || M < 1 || M % m) return IPT_ERR_INVALID_ARG;
    return ipt_100(d_ptr, 1, M / m, N, m, elem_bytes, d_workspace, ws_bytes, stream);
}

// -------------------------------------------------------------------- diagnostics
// ---------------------------------------------------------------- CUDA graphs
// A plan's launches (memsets + 1-3 kernels, or more for batches) captured once into an
// executable CUDA graph and replayed with one cudaGraphLaunch: no per-call host planning,
// validation or launch overhead (small matrices are launch-latency sensitive).  Capture
// runs on an internal stream; state built lazily on a first call (segment lists,
// self-resetting counters) is only used if it already exists -- transpose once before
// capturing to get the same kernels as the uncaptured call.
struct GraphHandle {
    cudaGraphExec_t exec;
    void *ws;   // workspace owned by the graph (freed by ipt_graph_destroy), or nullptr
};

ipt_status ipt_graph_create(void *d_base, int64_t count, int64_t stride_bytes, const ipt_plan_t *plan,
                            void *d_workspace, size_t ws_bytes, void **out) {
    if (!out) return IPT_ERR_INVALID_ARG;
    *out = nullptr;
    ipt_status s = validate_plan(plan);
    if (s) return s;
    if (count < 1) return IPT_ERR_INVALID_ARG;
    if ((s = check_ptr(d_base, plan->elem_bytes))) return s;
    const int64_t mat = plan->M * plan->N * plan->elem_bytes;
    if (count == 1) stride_bytes = mat;
    if (count > 1 && (stride_bytes < mat || stride_bytes % plan->elem_bytes)) return IPT_ERR_INVALID_ARG;
    const int device = current_device();
    if (device < 0) return IPT_ERR_NO_DEVICE;
    const size_t need = batched_ws(plan, count);
    if (d_workspace && ws_bytes < need) return IPT_ERR_NO_MEMORY;
    // without a caller workspace the graph owns one (allocated here, outside the capture,
    // freed by ipt_graph_destroy): replays of this graph are ordered on the caller's stream
    // and never share it with direct calls or other graphs (allocation nodes inside the
    // graph -- what run_plan does for a caller's capture -- cost 0.2-1.4 ms per replay)
    void *own = nullptr;
    if (!d_workspace && need) {
        if (cudaMalloc(&own, need) != cudaSuccess) {
            cudaGetLastError();
            return IPT_ERR_NO_MEMORY;
        }
        d_workspace = own;
        ws_bytes = need;
    }
    cudaStream_t cs;
    cudaError_t e = cudaStreamCreateWithFlags(&cs, cudaStreamNonBlocking);
    if (e != cudaSuccess) {
        if (own) cudaFree(own);
        return cuda_status(e);
    }
    // library-owned per-stream counters are never used under capture (memset nodes instead)
    cudaGraph_t g = nullptr;
    e = cudaStreamBeginCapture(cs, cudaStreamCaptureModeThreadLocal);
    if (e == cudaSuccess) {
        s = run_plan((char *)d_base, count, stride_bytes, plan, d_workspace, ws_bytes, cs, nullptr);
        cudaError_t e2 = cudaStreamEndCapture(cs, &g);
        if (!s && e2 != cudaSuccess) e = e2;
    }
    GraphHandle *h = nullptr;
    if (!s && e == cudaSuccess) {
        h = new GraphHandle{};
        h->ws = own;
        e = cudaGraphInstantiate(&h->exec, g, 0);
        if (e != cudaSuccess) { delete h; h = nullptr; }
    }
    if (g) cudaGraphDestroy(g);
    cudaStreamDestroy(cs);   // nothing was launched on it: captured work lives in the graph
    if ((s || e != cudaSuccess) && own) cudaFree(own);
    if (s) return s;
    if (e != cudaSuccess) return cuda_status(e);
    *out = h;
    return IPT_OK;
}

ipt_status ipt_graph_launch(void *graph, void *stream) {
    if (!graph) return IPT_ERR_INVALID_ARG;
    return cuda_status(cudaGraphLaunch(((GraphHandle *)graph)->exec, (cudaStream_t)stream));
}

ipt_status ipt_graph_destroy(void *graph) {
    if (!graph) return IPT_OK;
    GraphHandle *h = (GraphHandle *)graph;
    cudaError_t e = cudaGraphExecDestroy(h->exec);
    if (h->ws) {   // the caller synchronised: no replay still uses it
        const cudaError_t f = cudaFree(h->ws);
        if (e == cudaSuccess) e = f;
    }
    delete h;
    return cuda_status(e);
}

const char *ipt_status_string(ipt_status s) {
    switch (s) {
        case IPT_OK: return "IPT_OK";
        case IPT_ERR_INVALID_ARG: return "IPT_ERR_INVALID_ARG";
        case IPT_ERR_UNSUPPORTED_ELEM: return "IPT_ERR_UNSUPPORTED_ELEM";
        case IPT_ERR_MISALIGNED: return "IPT_ERR_MISALIGNED";
        case IPT_ERR_NO_MEMORY: return "IPT_ERR_NO_MEMORY";
        case IPT_ERR_CUDA: return "IPT_ERR_CUDA";
        case IPT_ERR_NO_DEVICE: return "IPT_ERR_NO_DEVICE";
    }
    return "IPT_ERR_UNKNOWN";
}

uint64_t ipt_kernel_launch_count(void) { return g_launches.load(); }

const char *ipt_last_cuda_error(void) { return cudaGetErrorString(g_last_cuda); }

const char *ipt_version(void) { return "libipt 0.1 (sm_100a)"; }

// Diagnostic hook (not in the ABI): the kernel stage `stage` (0..2) of `plan` applied to
// `count` packed matrices at `d_base` launches ("identity", "cycle_global", "cycle_ua",
// "cycle_seg", "tile_group_tma", "square_swap_vec", ...), copied into buf.  Used by the
// bench to attribute per-stage event times to kernels (the roofline's dominant kernel).
int ipt__stage_kernel(const ipt_plan_t *plan, int64_t count, const void *d_base, int stage, char *buf,
                      int len) {
    if (validate_plan(plan) || stage < 0 || stage > 2 || !buf || len < 1 || count < 1) return -1;
    const int device = current_device();
    StageDesc sd[3];
    plan_stages(plan, (char *)d_base, count, plan->M * plan->N * plan->elem_bytes, sd);
    const char *name = "identity";
    switch (plan->variant[stage]) {
        case IPT_VAR_TILE_ONCHIP: name = tile_kernel_name(sd[stage], device); break;
        case IPT_VAR_SQUARE_SWAP: name = square_kernel_name(sd[stage]); break;
        case IPT_VAR_CYCLE_GLOBAL: name = cycle_kernel_name(sd[stage], device); break;
        default: break;
    }
    snprintf(buf, (size_t)len, "%s", name);
    return 0;
}

// Internal self-test hook (not in the ABI): the multiply-high division used by every
// kernel's index map, evaluated on the host.
uint64_t ipt__fastdiv(uint64_t n, uint64_t d) { return fdiv(n, make_fastdiv(d)); }

uint32_t ipt__fastdiv32(uint32_t n, uint32_t d) {
    FastDiv32 f = make_fastdiv32(d);
    const uint32_t t = (uint32_t)(((uint64_t)n * f.m) >> 32);
    return (t + ((n - t) >> f.s1)) >> f.s2;
}

}  // extern "C"
