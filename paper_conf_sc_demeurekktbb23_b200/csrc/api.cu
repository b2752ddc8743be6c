// api.cu — the extern "C" boundary declared in include/toast_b200.h.
//
// Host side only: argument validation (before anything is launched), the per-device cache
// of encoded interval work lists, and dispatch to the kernel launchers.  No exception
// crosses the ABI; errors are returned as toast_status_t with a thread-local message.
#include <cuda_runtime.h>

#include <cstdarg>
#include <cstdio>
#include <cstring>
#include <mutex>
#include <string>
#include <vector>

#include "../../include/toast_b200.h"
#include "internal.h"

namespace toastb200 {

namespace {

thread_local std::string g_last_error;

int fail(int code, const char* fmt, ...) {
    char buf[512];
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(buf, sizeof(buf), fmt, ap);
    va_end(ap);
    g_last_error = buf;
    return code;
}

int ok() {
    g_last_error.clear();
    return TOAST_OK;
}

int cuda_fail(cudaError_t e, const char* where) {
    return fail(TOAST_ECUDA, "%s: %s", where, cudaGetErrorString(e));
}

// ---------------------------------------------------------------- interval work-list cache
//
// Work lists are cached per (device, chunk length, tail, interval set).  A new list is uploaded
// ASYNCHRONOUSLY on the caller's stream: stream-ordered allocation (cudaMallocAsync) and a
// cudaMemcpyAsync from a pinned host copy that the entry keeps until it is evicted, so a first
// call is as asynchronous as every later one (and capturable in a CUDA graph).  An event recorded
// after the upload orders launches on other streams after it.  The cache lock is held until the
// caller's launch has been enqueued (WorkListLease), so no other host thread can evict the entry
// in between; eviction (LRU, rare) synchronises the entry's event before freeing.

struct CacheEntry {
    int device;
    int chunk;
    int64_t tail;  // the last `tail` in-interval samples are cut into chunks of kTailChunk
    std::vector<toast_interval_t> intervals;
    Chunk* d_chunks;
    Chunk* h_pinned;  // pinned staging of the upload (kept until eviction)
    cudaEvent_t uploaded;
    cudaStream_t upload_stream;
    int64_t n_chunks;
    int64_t n_samples;
    uint64_t last_use;
};

std::mutex g_cache_mu;
std::vector<CacheEntry> g_cache;
uint64_t g_cache_clock = 0;
constexpr size_t kCacheMax = 256;

void free_entry(CacheEntry& c) {
    int cur = 0;
    cudaGetDevice(&cur);
    cudaSetDevice(c.device);
    if (c.uploaded) {
        cudaEventSynchronize(c.uploaded);
        cudaEventDestroy(c.uploaded);
    }
    if (c.d_chunks) cudaFree(c.d_chunks);
    if (c.h_pinned) cudaFreeHost(c.h_pinned);
    cudaSetDevice(cur);
}

int validate_intervals(const toast_interval_t* iv, int64_t n, int64_t n_samp) {
    if (n < 0) return fail(TOAST_EINVAL, "n_intervals < 0");
    if (n > 0 && !iv) return fail(TOAST_EINVAL, "intervals is NULL with n_intervals > 0");
    for (int64_t i = 0; i < n; ++i) {
        if (iv[i].first < 0 || iv[i].last >= n_samp || iv[i].last < iv[i].first - 1)
            return fail(TOAST_EINVAL, "interval %lld = [%lld, %lld] outside [0, n_samp=%lld)", (long long)i,
                        (long long)iv[i].first, (long long)iv[i].last, (long long)n_samp);
        if (i > 0 && iv[i].first <= iv[i - 1].last)
            return fail(TOAST_EINVAL, "intervals %lld and %lld overlap or are unsorted", (long long)(i - 1),
                        (long long)i);
    }
    return TOAST_OK;
}

// Chunk length of the work-list tail (see fused_worklist).
#ifndef TB_TAIL_CHUNK
#define TB_TAIL_CHUNK 32
#endif
#ifndef TB_TAIL_ITEMS
#define TB_TAIL_ITEMS 4  // tail items per resident warp (measured best of 2/4/8: C2 -3.7 %, C3 -2.7 % vs 2)
#endif
constexpr int kTailChunk = TB_TAIL_CHUNK;

// A work list valid while the lease (and so the cache lock) lives: enqueue the launch, then let
// the lease go.
struct WorkListLease {
    WorkList wl;
    std::unique_lock<std::mutex> lock;
};

// Chunks of `chunk` samples that never cross an interval and, inside an interval, end on
// multiples of 16 samples (the fused kernel's TMA boxes), so only interval edges give partial
// 16-sample blocks; the last `tail` in-interval samples in chunks of kTailChunk.
std::vector<Chunk> build_chunks(const toast_interval_t* iv, int64_t n, int chunk, int64_t tail, int64_t* total_out) {
    std::vector<Chunk> chunks;
    int64_t all = 0;
    for (int64_t i = 0; i < n; ++i) all += iv[i].last - iv[i].first + 1;
    int64_t total = 0;
    for (int64_t i = 0; i < n; ++i) {
        for (int64_t f = iv[i].first; f <= iv[i].last;) {
            const int len = (total >= all - tail) ? kTailChunk : chunk;
            int64_t end = f + len;
            if ((len & 15) == 0 && (end & ~int64_t(15)) > f) end &= ~int64_t(15);
            const int64_t cnt = std::min<int64_t>(end - f, iv[i].last - f + 1);
            chunks.push_back(Chunk{f, (int32_t)cnt, (int32_t)i});
            total += cnt;
            f += cnt;
        }
    }
    *total_out = total;
    return chunks;
}

int get_worklist(const toast_interval_t* iv, int64_t n, int64_t n_samp, cudaStream_t st, WorkListLease* out,
                 int chunk = kChunk, int64_t tail = 0) {
    int rc = validate_intervals(iv, n, n_samp);
    if (rc != TOAST_OK) return rc;
    int dev = 0;
    cudaError_t e = cudaGetDevice(&dev);
    if (e != cudaSuccess) return cuda_fail(e, "cudaGetDevice");
    std::unique_lock<std::mutex> lk(g_cache_mu);
    for (auto& c : g_cache) {
        if (c.device == dev && c.chunk == chunk && c.tail == tail && (int64_t)c.intervals.size() == n &&
            (n == 0 || std::memcmp(c.intervals.data(), iv, sizeof(toast_interval_t) * n) == 0)) {
            c.last_use = ++g_cache_clock;
            if (c.uploaded && st != c.upload_stream) {
                // (a capturing stream may not wait on uncaptured work: CUDA-graph capture of a call
                // requires a prior call with the same intervals, synchronised — e.g. a warm-up)
                cudaStreamCaptureStatus cap = cudaStreamCaptureStatusNone;
                e = cudaStreamIsCapturing(st, &cap);
                if (e == cudaSuccess && cap == cudaStreamCaptureStatusNone) e = cudaStreamWaitEvent(st, c.uploaded, 0);
                if (e != cudaSuccess) return cuda_fail(e, "ordering after the work-list upload");
            }
            out->wl = WorkList{c.d_chunks, c.n_chunks, c.n_samples};
            out->lock = std::move(lk);
            return TOAST_OK;
        }
    }
    int64_t total = 0;
    std::vector<Chunk> chunks = build_chunks(iv, n, chunk, tail, &total);
    CacheEntry ce{dev, chunk, tail, std::vector<toast_interval_t>(iv, iv + n), nullptr, nullptr, nullptr, st,
                  (int64_t)chunks.size(), total, ++g_cache_clock};
    if (!chunks.empty()) {
        const size_t bytes = sizeof(Chunk) * chunks.size();
        e = cudaMallocHost(&ce.h_pinned, bytes);
        if (e != cudaSuccess) {
            cudaGetLastError();
            return fail(TOAST_ENOMEM, "cudaMallocHost of the work-list staging: %s", cudaGetErrorString(e));
        }
        std::memcpy(ce.h_pinned, chunks.data(), bytes);
        e = cudaMallocAsync(reinterpret_cast<void**>(&ce.d_chunks), bytes, st);
        if (e == cudaSuccess) e = cudaMemcpyAsync(ce.d_chunks, ce.h_pinned, bytes, cudaMemcpyHostToDevice, st);
        if (e == cudaSuccess) e = cudaEventCreateWithFlags(&ce.uploaded, cudaEventDisableTiming);
        if (e == cudaSuccess) e = cudaEventRecord(ce.uploaded, st);
        if (e != cudaSuccess) {
            cudaGetLastError();
            free_entry(ce);
            return fail(TOAST_ENOMEM, "work-list upload: %s", cudaGetErrorString(e));
        }
    }
    if (g_cache.size() >= kCacheMax) {  // evict the least recently used entry
        size_t lru = 0;
        for (size_t i = 1; i < g_cache.size(); ++i)
            if (g_cache[i].last_use < g_cache[lru].last_use) lru = i;
        free_entry(g_cache[lru]);
        g_cache.erase(g_cache.begin() + (long)lru);
    }
    g_cache.push_back(std::move(ce));
    const CacheEntry& c = g_cache.back();
    out->wl = WorkList{c.d_chunks, c.n_chunks, c.n_samples};
    out->lock = std::move(lk);
    return TOAST_OK;
}

// Work list of the fused kernels: chunks of kFusedChunk samples, shorter when few detector groups
// x few samples would leave the persistent grid idle (C1: 4 detectors, one group of 32 lanes),
// so that there are at least ~4 items per resident warp.  Items are handed out in list order,
// so the LAST items set the kernel's tail: the last TB_TAIL_ITEMS items' worth of samples per
// resident warp are cut into kTailChunk-sample chunks.  Only the final list is built and cached.
int fused_worklist(const toast_interval_t* iv, int64_t n, int64_t n_samp, int64_t n_det, int64_t nside,
                   cudaStream_t st, WorkListLease* out) {
    int rc = validate_intervals(iv, n, n_samp);
    if (rc != TOAST_OK) return rc;
    int64_t n_samples = 0;
    for (int64_t i = 0; i < n; ++i) n_samples += iv[i].last - iv[i].first + 1;
    const int64_t groups = (n_det + 31) / 32, warps = (int64_t)num_sms() * 16, want = 4 * warps;
    // large focal planes (>= 64 detector groups) on fine maps (nside >= 4096: C5) take 64-sample
    // chunks: the warps in flight then span half the time window, so the map lines they scatter
    // into are reused more in L2 (C5 2.57 -> 2.46 ms); at nside 2048 (C4) the longer chunks win
    // (fewer item switches and full-arctangent restarts: C4 46.4 -> 45.6 ms, r02p8)
#ifndef TB_FINE_MAP_CHUNK
#define TB_FINE_MAP_CHUNK (kFusedChunk / 2)  // C5 (r02fm): 64 2.479 ms, 48 2.498, 32 2.659
#endif
    int chunk = (groups >= 64 && nside >= 4096) ? TB_FINE_MAP_CHUNK : kFusedChunk;
    while (chunk > 16 && (n_samples / chunk) * groups < want) chunk /= 2;
#ifndef TB_NO_TAIL
    const int64_t tail =
        chunk > kTailChunk ? std::min<int64_t>(n_samples / 4, TB_TAIL_ITEMS * warps * kTailChunk / std::max<int64_t>(groups, 1)) : 0;
#else
    const int64_t tail = 0;
#endif
    return get_worklist(iv, n, n_samp, st, out, chunk, tail);
}

bool is_pow2(int64_t x) { return x > 0 && (x & (x - 1)) == 0; }

int check_nside(int64_t nside) {
    if (!is_pow2(nside) || nside > (int64_t(1) << 29))
        return fail(TOAST_EINVAL, "nside = %lld is not a power of two in [1, 2^29]", (long long)nside);
    return TOAST_OK;
}

int check_submap(int64_t n_pix_submap, int64_t npix) {
    if (n_pix_submap <= 0) return fail(TOAST_EINVAL, "n_pix_submap = %lld <= 0", (long long)n_pix_submap);
    if (npix > 0 && npix % n_pix_submap != 0)
        return fail(TOAST_EINVAL, "n_pix_submap = %lld does not divide npix = %lld", (long long)n_pix_submap,
                    (long long)npix);
    return TOAST_OK;
}

// The fused kernels index samples, chunks and work items with 32-bit integers.
int check_fused_dims(int64_t n_det, int64_t n_samp) {
    if (n_samp >= (int64_t(1) << 31))
        return fail(TOAST_EUNSUPPORTED, "n_samp = %lld >= 2^31 in one call (split the observation)", (long long)n_samp);
    if (n_det >= (int64_t(1) << 31)) return fail(TOAST_EUNSUPPORTED, "n_det = %lld >= 2^31", (long long)n_det);
    return TOAST_OK;
}

MapGeom make_map_geom(const int64_t* g2l, int64_t nps) {
    MapGeom m;
    m.global2local = g2l;
    m.n_pix_submap = nps;
    m.sm_shift = -1;
    if (is_pow2(nps)) {
        int sh = 0;
        while ((int64_t(1) << sh) < nps) ++sh;
        m.sm_shift = sh;
    }
    return m;
}

#define REQUIRE(ptr)                                                                 \
    do {                                                                             \
        if (!(ptr)) return fail(TOAST_EINVAL, "%s: required pointer " #ptr " is NULL", __func__); \
    } while (0)

#define REQUIRE_DIMS(n_det, n_samp)                                                                    \
    do {                                                                                               \
        if ((n_det) < 0 || (n_samp) < 0)                                                               \
            return fail(TOAST_EINVAL, "%s: n_det = %lld, n_samp = %lld must be >= 0", __func__,        \
                        (long long)(n_det), (long long)(n_samp));                                      \
    } while (0)

}  // namespace

// Per-device pool of work-distribution counters, handed out round robin so that launches
// in flight on different streams use different counters.
unsigned long long* sched_counter(int* err) {
    constexpr int kPool = 64;
    static std::mutex mu;
    static unsigned long long* pools[64] = {nullptr};
    static unsigned next[64] = {0};
    int dev = 0;
    if (cudaGetDevice(&dev) != cudaSuccess || dev < 0 || dev >= 64) {
        *err = 1;
        return nullptr;
    }
    std::lock_guard<std::mutex> lk(mu);
    if (!pools[dev]) {
        if (cudaMalloc(&pools[dev], kPool * 128) != cudaSuccess) {  // one 128-B line per counter
            cudaGetLastError();
            *err = 1;
            return nullptr;
        }
        cudaMemset(pools[dev], 0, kPool * 128);
    }
    *err = 0;
    return pools[dev] + (next[dev]++ % kPool) * (128 / sizeof(unsigned long long));
}

void release_offset_cache();

int num_sms() {
    static int sms[64] = {0};
    int dev = 0;
    cudaGetDevice(&dev);
    if (dev < 0 || dev >= 64) return 148;
    if (sms[dev] == 0) {
        int v = 0;
        if (cudaDeviceGetAttribute(&v, cudaDevAttrMultiProcessorCount, dev) != cudaSuccess || v <= 0) v = 148;
        sms[dev] = v;
    }
    return sms[dev];
}

}  // namespace toastb200

using namespace toastb200;

extern "C" {

const char* toast_last_error(void) { return g_last_error.c_str(); }

const char* toast_version(void) { return "toastb200 0.1.0 (sm_100a)"; }

const char* toast_last_fused_path(void) { return last_fused_path(); }

int toast_release(void) {
    {
        std::lock_guard<std::mutex> lk(g_cache_mu);
        for (auto& c : g_cache) free_entry(c);
        g_cache.clear();
    }
    release_offset_cache();
    return ok();
}

int toast_pointing_detector(const double* fp_quats, const double* boresight, const int32_t* quat_index,
                            double* quats, const toast_interval_t* intervals, int64_t n_intervals,
                            const uint8_t* shared_flags, uint8_t shared_flag_mask, int64_t n_det, int64_t n_samp,
                            void* stream) {
    REQUIRE_DIMS(n_det, n_samp);
    if (n_det > 0 && n_intervals > 0) {
        REQUIRE(fp_quats);
        REQUIRE(boresight);
        REQUIRE(quats);
    }
    WorkListLease lease;
    int rc = get_worklist(intervals, n_intervals, n_samp, (cudaStream_t)stream, &lease);
    if (rc != TOAST_OK) return rc;
    cudaError_t e = launch_pointing_detector(lease.wl, fp_quats, boresight, quat_index, quats, shared_flags,
                                             shared_flag_mask, n_det, n_samp, (cudaStream_t)stream);
    if (e != cudaSuccess) return cuda_fail(e, "pointing_detector launch");
    return ok();
}

int toast_pixels_healpix(const int32_t* quat_index, const double* quats, const uint8_t* shared_flags,
                         uint8_t shared_flag_mask, const int32_t* pixel_index, int64_t* pixels,
                         const toast_interval_t* intervals, int64_t n_intervals, uint8_t* hit_submaps,
                         int64_t n_pix_submap, int64_t nside, int nest, int64_t n_det, int64_t n_samp,
                         void* stream) {
    REQUIRE_DIMS(n_det, n_samp);
    int rc = check_nside(nside);
    if (rc != TOAST_OK) return rc;
    if (nest != 0 && nest != 1) return fail(TOAST_EINVAL, "nest = %d must be 0 (RING) or 1 (NESTED)", nest);
    rc = check_submap(n_pix_submap, 12 * nside * nside);
    if (rc != TOAST_OK) return rc;
    if (n_det > 0 && n_intervals > 0) {
        REQUIRE(quats);
        REQUIRE(pixels);
    }
    WorkListLease lease;
    rc = get_worklist(intervals, n_intervals, n_samp, (cudaStream_t)stream, &lease);
    if (rc != TOAST_OK) return rc;
    cudaError_t e = launch_pixels_healpix(lease.wl, quat_index, quats, shared_flags, shared_flag_mask, pixel_index, pixels,
                                          hit_submaps, n_pix_submap, nside, nest, n_det, n_samp,
                                          (cudaStream_t)stream);
    if (e != cudaSuccess) return cuda_fail(e, "pixels_healpix launch");
    return ok();
}

int toast_stokes_weights_iqu_ex(const int32_t* quat_index, const double* quats, const int32_t* weight_index,
                                double* weights, const double* hwp, const double* epsilon, const double* gamma, int iau,
                                double cal, const toast_interval_t* intervals, int64_t n_intervals, int64_t n_det,
                                int64_t n_samp, void* stream) {
    REQUIRE_DIMS(n_det, n_samp);
    if (iau != 0 && iau != 1) return fail(TOAST_EINVAL, "iau = %d must be 0 or 1", iau);
    if (n_det > 0 && n_intervals > 0) {
        REQUIRE(quats);
        REQUIRE(weights);
        REQUIRE(epsilon);
    }
    WorkListLease lease;
    int rc = get_worklist(intervals, n_intervals, n_samp, (cudaStream_t)stream, &lease);
    if (rc != TOAST_OK) return rc;
    cudaError_t e = launch_stokes_weights_iqu(lease.wl, quat_index, quats, weight_index, weights, hwp, epsilon, cal,
                                              n_det, n_samp, (cudaStream_t)stream, gamma, iau);
    if (e != cudaSuccess) return cuda_fail(e, "stokes_weights_iqu launch");
    return ok();
}

int toast_stokes_weights_iqu(const int32_t* quat_index, const double* quats, const int32_t* weight_index,
                             double* weights, const double* hwp, const double* epsilon, double cal,
                             const toast_interval_t* intervals, int64_t n_intervals, int64_t n_det, int64_t n_samp,
                             void* stream) {
    return toast_stokes_weights_iqu_ex(quat_index, quats, weight_index, weights, hwp, epsilon, nullptr, 0, cal,
                                       intervals, n_intervals, n_det, n_samp, stream);
}

int toast_build_noise_weighted(const int64_t* global2local, double* zmap, int64_t n_pix_submap, int64_t nnz,
                               const int32_t* pixel_index, const int64_t* pixels, const int32_t* weight_index,
                               const double* weights, const int32_t* data_index, const double* det_data,
                               const int32_t* flag_index, const uint8_t* det_flags, uint8_t det_flag_mask,
                               const double* det_scale, const uint8_t* shared_flags, uint8_t shared_flag_mask,
                               const toast_interval_t* intervals, int64_t n_intervals, int64_t n_det, int64_t n_samp,
                               void* stream) {
    REQUIRE_DIMS(n_det, n_samp);
    if (nnz != 1 && nnz != 3) return fail(TOAST_EINVAL, "nnz = %lld must be 1 or 3", (long long)nnz);
    int rc = check_submap(n_pix_submap, 0);
    if (rc != TOAST_OK) return rc;
    if (n_det > 0 && n_intervals > 0) {
        REQUIRE(global2local);
        REQUIRE(zmap);
        REQUIRE(pixels);
        REQUIRE(weights);
        REQUIRE(det_data);
        REQUIRE(det_scale);
    }
    WorkListLease lease;
    rc = get_worklist(intervals, n_intervals, n_samp, (cudaStream_t)stream, &lease);
    if (rc != TOAST_OK) return rc;
    cudaError_t e = launch_build_noise_weighted(lease.wl, make_map_geom(global2local, n_pix_submap), zmap, (int)nnz,
                                                pixel_index, pixels, weight_index, weights, data_index, det_data,
                                                flag_index, det_flags, det_flag_mask, det_scale, shared_flags,
                                                shared_flag_mask, n_det, n_samp, (cudaStream_t)stream);
    if (e != cudaSuccess) return cuda_fail(e, "build_noise_weighted launch");
    return ok();
}

int toast_scan_map(const int64_t* global2local, int64_t n_pix_submap, const double* mapdata, int64_t nnz,
                   const int32_t* data_index, double* det_data, const int32_t* pixel_index, const int64_t* pixels,
                   const int32_t* weight_index, const double* weights, const toast_interval_t* intervals,
                   int64_t n_intervals, double data_scale, int should_zero, int should_subtract, int64_t n_det,
                   int64_t n_samp, void* stream) {
    REQUIRE_DIMS(n_det, n_samp);
    if (nnz != 1 && nnz != 3) return fail(TOAST_EINVAL, "nnz = %lld must be 1 or 3", (long long)nnz);
    int rc = check_submap(n_pix_submap, 0);
    if (rc != TOAST_OK) return rc;
    if (n_det > 0 && n_intervals > 0) {
        REQUIRE(global2local);
        REQUIRE(mapdata);
        REQUIRE(det_data);
        REQUIRE(pixels);
        REQUIRE(weights);
    }
    WorkListLease lease;
    rc = get_worklist(intervals, n_intervals, n_samp, (cudaStream_t)stream, &lease);
    if (rc != TOAST_OK) return rc;
    cudaError_t e = launch_scan_map(lease.wl, make_map_geom(global2local, n_pix_submap), mapdata, (int)nnz, data_index,
                                    det_data, pixel_index, pixels, weight_index, weights, data_scale, should_zero,
                                    should_subtract, n_det, n_samp, (cudaStream_t)stream);
    if (e != cudaSuccess) return cuda_fail(e, "scan_map launch");
    return ok();
}

int toast_pointing_to_map_ex(const double* fp_quats, const double* boresight, const double* hwp,
                             const double* epsilon, double cal, const double* det_scale, const double* det_data,
                             const uint8_t* det_flags, uint8_t det_flag_mask, const uint8_t* shared_flags,
                             uint8_t shared_flag_mask, const toast_interval_t* intervals, int64_t n_intervals,
                             int64_t nside, int nest, int64_t nnz, const int64_t* global2local, int64_t n_pix_submap,
                             void* zmap, uint8_t* hit_submaps, int64_t* pixels_out, double* weights_out, int64_t n_det,
                             int64_t n_samp, const toast_map_options_t* opts, void* stream) {
    REQUIRE_DIMS(n_det, n_samp);
    int rc = check_nside(nside);
    if (rc != TOAST_OK) return rc;
    if (nest != 0 && nest != 1) return fail(TOAST_EINVAL, "nest = %d must be 0 (RING) or 1 (NESTED)", nest);
    if (nnz != 1 && nnz != 3) return fail(TOAST_EINVAL, "nnz = %lld must be 1 or 3", (long long)nnz);
    rc = check_submap(n_pix_submap, 12 * nside * nside);
    if (rc != TOAST_OK) return rc;
    rc = check_fused_dims(n_det, n_samp);
    if (rc != TOAST_OK) return rc;
    if (n_det > 0 && n_intervals > 0) {
        REQUIRE(fp_quats);
        REQUIRE(boresight);
        REQUIRE(epsilon);
        REQUIRE(det_scale);
        REQUIRE(det_data);
        REQUIRE(global2local);
        REQUIRE(zmap);
    }
    if (opts && opts->map_f32 && (pixels_out || weights_out))
        return fail(TOAST_EINVAL, "debug outputs are not available with an fp32 map");
    WorkListLease lease;
    rc = fused_worklist(intervals, n_intervals, n_samp, n_det, nside, (cudaStream_t)stream, &lease);
    if (rc != TOAST_OK) return rc;
    if ((int64_t)lease.wl.n_chunks * ((n_det + 31) / 32) >= (int64_t(1) << 31))
        return fail(TOAST_EUNSUPPORTED, "more than 2^31 work items (split the call over detectors)");
    FusedArgs a = {};
    a.fp_quats = fp_quats;
    a.boresight = boresight;
    a.hwp = hwp;
    a.epsilon = epsilon;
    a.cal = cal;
    a.det_scale = det_scale;
    a.det_data = det_data;
    a.det_flags = det_flags;
    a.det_flag_mask = det_flag_mask;
    a.shared_flags = shared_flags;
    a.shared_flag_mask = shared_flag_mask;
    a.nside = nside;
    a.nest = nest;
    a.nnz = (int)nnz;
    a.map = make_map_geom(global2local, n_pix_submap);
    a.zmap = static_cast<double*>(zmap);
    a.hit_submaps = hit_submaps;
    a.pixels_out = pixels_out;
    a.weights_out = weights_out;
    a.n_det = n_det;
    a.n_samp = n_samp;
    if (opts) {
        a.gamma = opts->gamma;
        a.iau = opts->iau;
        a.map_f32 = opts->map_f32;
        a.dropped = opts->dropped;
    }
    int serr = 0;
    unsigned long long* sched = sched_counter(&serr);
    if (serr) return fail(TOAST_ENOMEM, "could not allocate the work-distribution counter");
    cudaError_t e = launch_pointing_to_map(lease.wl, a, sched, (cudaStream_t)stream);
    if (e != cudaSuccess) return cuda_fail(e, "pointing_to_map launch");
    return ok();
}

int toast_pointing_to_map(const double* fp_quats, const double* boresight, const double* hwp, const double* epsilon,
                          double cal, const double* det_scale, const double* det_data, const uint8_t* det_flags,
                          uint8_t det_flag_mask, const uint8_t* shared_flags, uint8_t shared_flag_mask,
                          const toast_interval_t* intervals, int64_t n_intervals, int64_t nside, int nest,
                          int64_t nnz, const int64_t* global2local, int64_t n_pix_submap, double* zmap,
                          uint8_t* hit_submaps, int64_t* pixels_out, double* weights_out, int64_t n_det,
                          int64_t n_samp, void* stream) {
    return toast_pointing_to_map_ex(fp_quats, boresight, hwp, epsilon, cal, det_scale, det_data, det_flags,
                                    det_flag_mask, shared_flags, shared_flag_mask, intervals, n_intervals, nside, nest,
                                    nnz, global2local, n_pix_submap, zmap, hit_submaps, pixels_out, weights_out, n_det,
                                    n_samp, nullptr, stream);
}

}  // extern "C"

extern "C" int toast_pointing_to_tod_ex(const double* fp_quats, const double* boresight, const double* hwp,
                                        const double* epsilon, double cal, const uint8_t* shared_flags,
                                        uint8_t shared_flag_mask, const toast_interval_t* intervals,
                                        int64_t n_intervals, int64_t nside, int nest, int64_t nnz,
                                        const int64_t* global2local, int64_t n_pix_submap, const void* mapdata,
                                        double data_scale, int should_zero, int should_subtract, double* det_data,
                                        int64_t n_det, int64_t n_samp, const toast_map_options_t* opts, void* stream) {
    using namespace toastb200;
    REQUIRE_DIMS(n_det, n_samp);
    int rc = check_nside(nside);
    if (rc != TOAST_OK) return rc;
    if (nest != 0 && nest != 1) return fail(TOAST_EINVAL, "nest = %d must be 0 (RING) or 1 (NESTED)", nest);
    if (nnz != 1 && nnz != 3) return fail(TOAST_EINVAL, "nnz = %lld must be 1 or 3", (long long)nnz);
    rc = check_submap(n_pix_submap, 12 * nside * nside);
    if (rc != TOAST_OK) return rc;
    rc = check_fused_dims(n_det, n_samp);
    if (rc != TOAST_OK) return rc;
    if (n_det > 0 && n_intervals > 0) {
        REQUIRE(fp_quats);
        REQUIRE(boresight);
        REQUIRE(epsilon);
        REQUIRE(global2local);
        REQUIRE(mapdata);
        REQUIRE(det_data);
    }
    if (opts && opts->dropped) return fail(TOAST_EINVAL, "the dropped-sample counter applies to pointing_to_map only");
    WorkListLease lease;
    rc = fused_worklist(intervals, n_intervals, n_samp, n_det, nside, (cudaStream_t)stream, &lease);
    if (rc != TOAST_OK) return rc;
    if ((int64_t)lease.wl.n_chunks * ((n_det + 31) / 32) >= (int64_t(1) << 31))
        return fail(TOAST_EUNSUPPORTED, "more than 2^31 work items (split the call over detectors)");
    FusedArgs a = {};
    a.fp_quats = fp_quats;
    a.boresight = boresight;
    a.hwp = hwp;
    a.epsilon = epsilon;
    a.cal = cal;
    a.det_scale = epsilon;  // unused by the scan; any valid [n_det] array
    a.det_data = det_data;
    a.shared_flags = shared_flags;
    a.shared_flag_mask = shared_flag_mask;
    a.nside = nside;
    a.nest = nest;
    a.nnz = (int)nnz;
    a.map = make_map_geom(global2local, n_pix_submap);
    a.n_det = n_det;
    a.n_samp = n_samp;
    a.mapdata = static_cast<const double*>(mapdata);
    a.data_scale = data_scale;
    a.should_zero = should_zero;
    a.should_subtract = should_subtract;
    a.tod_out = det_data;
    if (opts) {
        a.gamma = opts->gamma;
        a.iau = opts->iau;
        a.map_f32 = opts->map_f32;
    }
    int serr = 0;
    unsigned long long* sched = sched_counter(&serr);
    if (serr) return fail(TOAST_ENOMEM, "could not allocate the work-distribution counter");
    cudaError_t e = launch_pointing_to_tod(lease.wl, a, sched, (cudaStream_t)stream);
    if (e != cudaSuccess) return cuda_fail(e, "pointing_to_tod launch");
    return ok();
}

extern "C" int toast_pointing_to_tod(const double* fp_quats, const double* boresight, const double* hwp,
                                     const double* epsilon, double cal, const uint8_t* shared_flags,
                                     uint8_t shared_flag_mask, const toast_interval_t* intervals, int64_t n_intervals,
                                     int64_t nside, int nest, int64_t nnz, const int64_t* global2local,
                                     int64_t n_pix_submap, const double* mapdata, double data_scale, int should_zero,
                                     int should_subtract, double* det_data, int64_t n_det, int64_t n_samp,
                                     void* stream) {
    return toast_pointing_to_tod_ex(fp_quats, boresight, hwp, epsilon, cal, shared_flags, shared_flag_mask, intervals,
                                    n_intervals, nside, nest, nnz, global2local, n_pix_submap, mapdata, data_scale,
                                    should_zero, should_subtract, det_data, n_det, n_samp, nullptr, stream);
}

// ---------------------------------------------------------------- NEXT rows (f2, f4)

namespace toastb200 {
namespace {

struct OffsetCacheEntry {
    int device;
    int step;
    std::vector<toast_interval_t> intervals;
    int64_t* d_arrays;  // [2][n]: iv_first, view_base
    int64_t* h_pinned;  // pinned staging of the upload (kept until eviction)
    cudaEvent_t uploaded;
    cudaStream_t upload_stream;
    uint64_t last_use;
};
std::mutex g_ocache_mu;
std::vector<OffsetCacheEntry> g_ocache;
uint64_t g_ocache_clock = 0;

void free_oentry(OffsetCacheEntry& c) {
    int cur = 0;
    cudaGetDevice(&cur);
    cudaSetDevice(c.device);
    if (c.uploaded) {
        cudaEventSynchronize(c.uploaded);
        cudaEventDestroy(c.uploaded);
    }
    if (c.d_arrays) cudaFree(c.d_arrays);
    if (c.h_pinned) cudaFreeHost(c.h_pinned);
    cudaSetDevice(cur);
}

// Offset views of an interval set, uploaded asynchronously on the caller's stream like the work
// lists (the lock is held through the caller's launch by the lease).
int get_offset_views(const toast_interval_t* iv, int64_t n, int64_t step, cudaStream_t st, OffsetViews* out,
                     std::unique_lock<std::mutex>* lease) {
    if (step < 1 || step > (int64_t(1) << 30)) return fail(TOAST_EINVAL, "step_length = %lld must be in [1, 2^30]",
                                                           (long long)step);
    int dev = 0;
    cudaError_t e = cudaGetDevice(&dev);
    if (e != cudaSuccess) return cuda_fail(e, "cudaGetDevice");
    std::unique_lock<std::mutex> lk(g_ocache_mu);
    for (auto& c : g_ocache) {
        if (c.device == dev && c.step == (int)step && (int64_t)c.intervals.size() == n &&
            (n == 0 || std::memcmp(c.intervals.data(), iv, sizeof(toast_interval_t) * n) == 0)) {
            c.last_use = ++g_ocache_clock;
            if (c.uploaded && st != c.upload_stream) {
                // (a capturing stream may not wait on uncaptured work: CUDA-graph capture of a call
                // requires a prior call with the same intervals, synchronised — e.g. a warm-up)
                cudaStreamCaptureStatus cap = cudaStreamCaptureStatusNone;
                e = cudaStreamIsCapturing(st, &cap);
                if (e == cudaSuccess && cap == cudaStreamCaptureStatusNone) e = cudaStreamWaitEvent(st, c.uploaded, 0);
                if (e != cudaSuccess) return cuda_fail(e, "ordering after the offset-view upload");
            }
            *out = OffsetViews{c.d_arrays, c.d_arrays + n, (int)step};
            *lease = std::move(lk);
            return TOAST_OK;
        }
    }
    const size_t cnt = 2 * (size_t)std::max<int64_t>(n, 1);
    OffsetCacheEntry ce{dev, (int)step, std::vector<toast_interval_t>(iv, iv + n), nullptr, nullptr, nullptr, st,
                        ++g_ocache_clock};
    e = cudaMallocHost(&ce.h_pinned, sizeof(int64_t) * cnt);
    if (e != cudaSuccess) {
        cudaGetLastError();
        return fail(TOAST_ENOMEM, "cudaMallocHost of the offset views: %s", cudaGetErrorString(e));
    }
    int64_t base = 0;
    ce.h_pinned[0] = ce.h_pinned[cnt - 1] = 0;
    for (int64_t i = 0; i < n; ++i) {
        ce.h_pinned[i] = iv[i].first;
        ce.h_pinned[n + i] = base;
        const int64_t len = iv[i].last - iv[i].first + 1;
        base += (len + step - 1) / step;
    }
    e = cudaMallocAsync(reinterpret_cast<void**>(&ce.d_arrays), sizeof(int64_t) * cnt, st);
    if (e == cudaSuccess) e = cudaMemcpyAsync(ce.d_arrays, ce.h_pinned, sizeof(int64_t) * cnt, cudaMemcpyHostToDevice, st);
    if (e == cudaSuccess) e = cudaEventCreateWithFlags(&ce.uploaded, cudaEventDisableTiming);
    if (e == cudaSuccess) e = cudaEventRecord(ce.uploaded, st);
    if (e != cudaSuccess) {
        cudaGetLastError();
        free_oentry(ce);
        return fail(TOAST_ENOMEM, "offset-view upload: %s", cudaGetErrorString(e));
    }
    if (g_ocache.size() >= kCacheMax) {
        size_t lru = 0;
        for (size_t i = 1; i < g_ocache.size(); ++i)
            if (g_ocache[i].last_use < g_ocache[lru].last_use) lru = i;
        free_oentry(g_ocache[lru]);
        g_ocache.erase(g_ocache.begin() + (long)lru);
    }
    g_ocache.push_back(std::move(ce));
    const OffsetCacheEntry& c = g_ocache.back();
    *out = OffsetViews{c.d_arrays, c.d_arrays + n, (int)step};
    *lease = std::move(lk);
    return TOAST_OK;
}

}  // namespace

void release_offset_cache() {
    std::lock_guard<std::mutex> lk(g_ocache_mu);
    for (auto& c : g_ocache) free_oentry(c);
    g_ocache.clear();
}

}  // namespace toastb200

extern "C" int toast_stokes_weights_i(const int32_t* weight_index, double* weights, double cal,
                                      const toast_interval_t* intervals, int64_t n_intervals, int64_t n_det,
                                      int64_t n_samp, void* stream) {
    using namespace toastb200;
    REQUIRE_DIMS(n_det, n_samp);
    if (n_det > 0 && n_intervals > 0) REQUIRE(weights);
    WorkListLease lease;
    int rc = get_worklist(intervals, n_intervals, n_samp, (cudaStream_t)stream, &lease);
    if (rc != TOAST_OK) return rc;
    cudaError_t e = launch_stokes_weights_i(lease.wl, weight_index, weights, cal, n_det, n_samp, (cudaStream_t)stream);
    if (e != cudaSuccess) return cuda_fail(e, "stokes_weights_i launch");
    return ok();
}

extern "C" int toast_noise_weight(const int32_t* data_index, double* det_data, const double* det_weights,
                                  const toast_interval_t* intervals, int64_t n_intervals, int64_t n_det, int64_t n_samp,
                                  void* stream) {
    using namespace toastb200;
    REQUIRE_DIMS(n_det, n_samp);
    if (n_det > 0 && n_intervals > 0) {
        REQUIRE(det_data);
        REQUIRE(det_weights);
    }
    WorkListLease lease;
    int rc = get_worklist(intervals, n_intervals, n_samp, (cudaStream_t)stream, &lease);
    if (rc != TOAST_OK) return rc;
    cudaError_t e = launch_noise_weight(lease.wl, data_index, det_data, det_weights, n_det, n_samp, (cudaStream_t)stream);
    if (e != cudaSuccess) return cuda_fail(e, "noise_weight launch");
    return ok();
}

extern "C" int toast_template_offset_add_to_signal(int64_t step_length, const int64_t* amp_offset,
                                                   const double* amplitudes, const int32_t* data_index,
                                                   double* det_data, const toast_interval_t* intervals,
                                                   int64_t n_intervals, int64_t n_det, int64_t n_samp, void* stream) {
    using namespace toastb200;
    REQUIRE_DIMS(n_det, n_samp);
    if (n_det > 0 && n_intervals > 0) {
        REQUIRE(amp_offset);
        REQUIRE(amplitudes);
        REQUIRE(det_data);
    }
    WorkListLease lease;
    int rc = get_worklist(intervals, n_intervals, n_samp, (cudaStream_t)stream, &lease);
    if (rc != TOAST_OK) return rc;
    OffsetViews v;
    std::unique_lock<std::mutex> vlease;
    rc = get_offset_views(intervals, n_intervals, step_length, (cudaStream_t)stream, &v, &vlease);
    if (rc != TOAST_OK) return rc;
    cudaError_t e = launch_offset_add(lease.wl, v, amp_offset, amplitudes, data_index, det_data, n_det, n_samp,
                                      (cudaStream_t)stream);
    if (e != cudaSuccess) return cuda_fail(e, "template_offset_add_to_signal launch");
    return ok();
}

extern "C" int toast_template_offset_project_signal(int64_t step_length, const int64_t* amp_offset, double* amplitudes,
                                                    const int32_t* data_index, const double* det_data,
                                                    const int32_t* flag_index, const uint8_t* det_flags,
                                                    uint8_t det_flag_mask, const toast_interval_t* intervals,
                                                    int64_t n_intervals, int64_t n_det, int64_t n_samp, void* stream) {
    using namespace toastb200;
    REQUIRE_DIMS(n_det, n_samp);
    if (n_det > 0 && n_intervals > 0) {
        REQUIRE(amp_offset);
        REQUIRE(amplitudes);
        REQUIRE(det_data);
    }
    WorkListLease lease;
    int rc = get_worklist(intervals, n_intervals, n_samp, (cudaStream_t)stream, &lease);
    if (rc != TOAST_OK) return rc;
    OffsetViews v;
    std::unique_lock<std::mutex> vlease;
    rc = get_offset_views(intervals, n_intervals, step_length, (cudaStream_t)stream, &v, &vlease);
    if (rc != TOAST_OK) return rc;
    cudaError_t e = launch_offset_project(lease.wl, v, amp_offset, amplitudes, data_index, det_data, flag_index, det_flags,
                                          det_flag_mask, n_det, n_samp, (cudaStream_t)stream);
    if (e != cudaSuccess) return cuda_fail(e, "template_offset_project_signal launch");
    return ok();
}

extern "C" int toast_template_offset_apply_diag_precond(const double* offset_var, const double* amp_in,
                                                        double* amp_out, int64_t n_amp, void* stream) {
    using namespace toastb200;
    if (n_amp < 0) return fail(TOAST_EINVAL, "n_amp = %lld < 0", (long long)n_amp);
    if (n_amp > 0) {
        REQUIRE(offset_var);
        REQUIRE(amp_in);
        REQUIRE(amp_out);
    }
    cudaError_t e = launch_precond(offset_var, amp_in, amp_out, n_amp, (cudaStream_t)stream);
    if (e != cudaSuccess) return cuda_fail(e, "template_offset_apply_diag_precond launch");
    return ok();
}

extern "C" int toast_map_allreduce_nvls(double* mc, int64_t n, unsigned* const* pads, int rank, int world,
                                        void* stream) {
    using namespace toastb200;
    if (n < 0) return fail(TOAST_EINVAL, "n = %lld < 0", (long long)n);
    if (world < 1 || rank < 0 || rank >= world)
        return fail(TOAST_EINVAL, "rank %d / world %d out of range", rank, world);
    if (n > 0 && !mc) return fail(TOAST_EINVAL, "mc is NULL");
    if (world > 1 && !pads) return fail(TOAST_EINVAL, "pads is NULL with world > 1");
    const cudaError_t e = launch_map_allreduce_nvls(mc, n, pads, rank, world, (cudaStream_t)stream);
    if (e != cudaSuccess) return cuda_fail(e, "map_allreduce_nvls launch");
    return ok();
}
