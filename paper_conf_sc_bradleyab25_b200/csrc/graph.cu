// graph.cu -- fsgc_load_graph: edge list -> deduplicated, symmetrised,
// degree-ordered CSR in HBM (north_star; Sec. 2 undirected simple
// graphs, Sec. 3.6 degree-based matching order / symmetry breaking on ids).
//
// Device pipeline (all on `stream`, sorts/compaction via CUB, the rest here):
//   1 emit    each input edge (a,b), a != b  ->  keys a<<B|b and b<<B|a
//             (B = bits to hold n-1); loops / out-of-range -> sentinel
//   2 sort    radix sort on the low 2B bits; 3 unique (dedup directed pairs)
//   4 degree  per-vertex lower_bound into the sorted keys
//   5 order   sort (deg<<B | id) -> new id = rank (degree asc, id asc)
//   6 relabel keys -> rank[a]<<B | rank[b]; radix sort again
//   7 CSR     adj/row = key halves, offsets = exclusive scan of new degrees,
//             oriented edges (u < v) = compaction of the upper triangle
// HBM layout of the result: offsets int64[n+1], adj int32[2m], row int32[2m],
// osrc/odst int32[m] (SoA, sorted by (u, v)), order int32[n].
#include <cub/cub.cuh>
#include <atomic>
#include <mutex>
#include <set>
#include <map>
#include <cstdlib>
#include <vector>
#include <algorithm>
#include "devbuf.cuh"

namespace {

__global__ void emit_keys(const void* __restrict__ edges, int64_t E, int ib, int64_t n, int B,
                          uint64_t sentinel, uint64_t* __restrict__ keys, int* __restrict__ bad) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < E;
         i += (int64_t)gridDim.x * blockDim.x) {
        int64_t a, b;
        if (ib == 4) {
            const int32_t* e = reinterpret_cast<const int32_t*>(edges);
            a = e[2 * i]; b = e[2 * i + 1];
        } else {
            const int64_t* e = reinterpret_cast<const int64_t*>(edges);
            a = e[2 * i]; b = e[2 * i + 1];
        }
        uint64_t k0 = sentinel, k1 = sentinel;
        if (a < 0 || b < 0 || a >= n || b >= n) {
            *bad = 1;
        } else if (a != b) {
            k0 = ((uint64_t)a << B) | (uint64_t)b;
            k1 = ((uint64_t)b << B) | (uint64_t)a;
        }
        keys[2 * i] = k0;
        keys[2 * i + 1] = k1;
    }
}

// offs[v] = first index i with (keys[i] >> B) >= v, for v in [0, n]
__global__ void lower_bounds(const uint64_t* __restrict__ keys, int64_t M, int64_t n, int B,
                             int64_t* __restrict__ offs) {
    for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v <= n;
         v += (int64_t)gridDim.x * blockDim.x) {
        uint64_t target = (uint64_t)v << B;
        int64_t lo = 0, hi = M;
        while (lo < hi) {
            int64_t mid = (lo + hi) >> 1;
            if (keys[mid] < target) lo = mid + 1; else hi = mid;
        }
        offs[v] = lo;
    }
}

__global__ void degree_keys(const int64_t* __restrict__ offs, int64_t n, int B, uint64_t* __restrict__ vk) {
    for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n;
         v += (int64_t)gridDim.x * blockDim.x)
        vk[v] = ((uint64_t)(offs[v + 1] - offs[v]) << B) | (uint64_t)v;
}

__global__ void ranks_from_order(const uint64_t* __restrict__ vk, int64_t n, int B,
                                 int32_t* __restrict__ order, int32_t* __restrict__ rank,
                                 int64_t* __restrict__ deg_new) {
    const uint64_t mask = (1ull << B) - 1;
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n;
         i += (int64_t)gridDim.x * blockDim.x) {
        uint64_t k = vk[i];
        int32_t v = (int32_t)(k & mask);
        order[i] = v;
        rank[v] = (int32_t)i;
        deg_new[i] = (int64_t)(k >> B);
    }
}

__global__ void relabel_keys(uint64_t* __restrict__ keys, int64_t M, int B, const int32_t* __restrict__ rank) {
    const uint64_t mask = (1ull << B) - 1;
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < M;
         i += (int64_t)gridDim.x * blockDim.x) {
        uint64_t k = keys[i];
        uint64_t a = (uint64_t)rank[k >> B], b = (uint64_t)rank[k & mask];
        keys[i] = (a << B) | b;
    }
}

__global__ void split_keys(const uint64_t* __restrict__ keys, int64_t M, int B,
                           int32_t* __restrict__ row, int32_t* __restrict__ adj) {
    const uint64_t mask = (1ull << B) - 1;
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < M;
         i += (int64_t)gridDim.x * blockDim.x) {
        uint64_t k = keys[i];
        row[i] = (int32_t)(k >> B);
        adj[i] = (int32_t)(k & mask);
    }
}

// split[v] = first CSR position in v's list holding a neighbour > v;
// out[v] = number of such neighbours (the degree-oriented out-degree)
__global__ void split_points(const int64_t* __restrict__ offs, const int32_t* __restrict__ adj, int64_t n,
                             int64_t* __restrict__ split, int64_t* __restrict__ out) {
    for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n;
         v += (int64_t)gridDim.x * blockDim.x) {
        int64_t lo = offs[v], hi = offs[v + 1];
        const int64_t end = hi;
        while (lo < hi) {
            int64_t mid = (lo + hi) >> 1;
            if (adj[mid] <= (int32_t)v) lo = mid + 1; else hi = mid;
        }
        split[v] = lo;
        out[v] = end - lo;
    }
}

// bitmap rows of the hub vertices [hub_base, n)
__global__ void hub_bitmaps(const int64_t* __restrict__ offs, const int32_t* __restrict__ adj, int64_t hub_base,
                            int64_t n, int64_t words, uint32_t* __restrict__ bits) {
    const int64_t beg = offs[hub_base], end = offs[n];
    for (int64_t i = beg + blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < end;
         i += (int64_t)gridDim.x * blockDim.x) {
        // row of entry i: binary search in offs over [hub_base, n)
        int64_t lo = hub_base, hi = n;
        while (hi - lo > 1) {
            int64_t mid = (lo + hi) >> 1;
            if (offs[mid] <= i) lo = mid; else hi = mid;
        }
        const int32_t x = adj[i];
        atomicOr(bits + (lo - hub_base) * words + (x >> 5), 1u << (x & 31));
    }
}

struct UpperTri {
    int B;
    uint64_t mask;
    __host__ __device__ bool operator()(const uint64_t& k) const { return (k >> B) < (k & mask); }
};

// merge-kernel work order: key = merge length out(u) + out(v) of oriented
// edge i (capped at 2^20 - 1), value = i; sorted, so the 32 lanes of a warp
// get roots of similar cost (degree-aware binning, north_star)
__global__ void support_work_keys(const int64_t* __restrict__ offs, const int64_t* __restrict__ split,
                                  const int32_t* __restrict__ osrc, const int32_t* __restrict__ odst, int64_t m,
                                  uint32_t* __restrict__ key, int32_t* __restrict__ idx) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < m;
         i += (int64_t)gridDim.x * blockDim.x) {
        const int u = osrc[i], v = odst[i];
        const int64_t w = (offs[u + 1] - split[u]) + (offs[v + 1] - split[v]);
        key[i] = (uint32_t)(w < (1 << 20) - 1 ? w : (1 << 20) - 1);
        idx[i] = (int32_t)i;
    }
}

// rev[i - oofs[b]] = oriented index of (a, b) for the in-entry a = adj[i] of
// row b: sorting the oriented edges (a, b), stored in (a, b) order, by
// (b, a) lists them in the in-entries' CSR order.  Keys b << B | a, values e.
__global__ void rev_keys(const int32_t* __restrict__ osrc, const int32_t* __restrict__ odst, int64_t m, int B,
                         uint64_t* __restrict__ key, int32_t* __restrict__ val) {
    for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < m;
         e += (int64_t)gridDim.x * blockDim.x) {
        key[e] = ((uint64_t)odst[e] << B) | (uint64_t)osrc[e];
        val[e] = (int32_t)e;
    }
}

// triangle-listing units per middle vertex b (cnt[n] = 0 for the scans):
// warp-table units ceil(in(b) / SEG) when 1 <= out(b) <= capw, block-table
// units ceil(in(b) / CHUNK) when out(b) > capw; maxout = max out(b) of a
// block-table middle (sizes the block tables)
__global__ void unit_counts(const int64_t* __restrict__ offs, const int64_t* __restrict__ split, int64_t n,
                            int64_t* __restrict__ cnt, int64_t* __restrict__ cnt_big, int64_t capw,
                            unsigned long long* maxout) {
    unsigned long long mx = 0;
    for (int64_t b = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; b <= n;
         b += (int64_t)gridDim.x * blockDim.x) {
        int64_t c = 0, cb = 0;
        if (b < n) {
            const int64_t in = split[b] - offs[b], out = offs[b + 1] - split[b];
            if (in >= 1 && out >= 1 && out <= capw) c = (in + FSGC_SUP_SEG - 1) / FSGC_SUP_SEG;
            if (in >= 1 && out > capw) {
                cb = (in + FSGC_SUP_CHUNK - 1) / FSGC_SUP_CHUNK;
                mx = mx > (unsigned long long)out ? mx : (unsigned long long)out;
            }
        }
        cnt[b] = c;
        cnt_big[b] = cb;
    }
    if (mx) atomicMax(maxout, mx);
}

__global__ void unit_fill(const int64_t* __restrict__ uofs, int64_t n, uint64_t* __restrict__ units) {
    for (int64_t b = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; b < n;
         b += (int64_t)gridDim.x * blockDim.x)
        for (int64_t k = uofs[b]; k < uofs[b + 1]; ++k) units[k] = ((uint64_t)b << 32) | (uint64_t)(k - uofs[b]);
}

__global__ void gather_uv(const int32_t* __restrict__ idx, const int32_t* __restrict__ osrc,
                          const int32_t* __restrict__ odst, int64_t m, int32_t* __restrict__ su,
                          int32_t* __restrict__ sv) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < m;
         i += (int64_t)gridDim.x * blockDim.x) {
        const int32_t e = idx[i];
        su[i] = osrc[e];
        sv[i] = odst[e];
    }
}

// number of unique keys without the trailing sentinel run (dnum[0] in, out)
__global__ void unique_count(const uint64_t* __restrict__ uniq, int64_t* dnum, uint64_t sentinel) {
    const int64_t nu = dnum[0];
    dnum[0] = (nu > 0 && uniq[nu - 1] == sentinel) ? nu - 1 : nu;
}

// out[0] = first v in [lo, n) with deg(v) >= mindeg (n if none), out[1] = deg(n-1)
__global__ void hub_search(const int64_t* __restrict__ offs, int64_t n, int64_t lo, int64_t mindeg,
                           int64_t* out) {
    int64_t hi = n;
    while (lo < hi) {
        const int64_t mid = (lo + hi) >> 1;
        if (offs[mid + 1] - offs[mid] >= mindeg) hi = mid; else lo = mid + 1;
    }
    out[0] = lo;
    out[1] = offs[n] - offs[n - 1];
}

int grid_for(int64_t work) {
    int64_t g = (work + 255) / 256;
    if (g > 148 * 32) g = 148 * 32;
    if (g < 1) g = 1;
    return (int)g;
}

}  // namespace

// The build's temporaries (and the graph arrays) come from a private
// stream-ordered pool per device.  Its release threshold keeps up to
// FSGC_POOL_KEEP_BYTES (default 8 GiB) of freed pages mapped, so a load that
// follows a free (the e2e loop) does not map them again; the device's default
// pool -- which other libraries in the process may use -- is left untouched.
cudaMemPool_t fsgc_device_pool() {
    static std::mutex mu;
    static std::map<int, cudaMemPool_t> pools;
    int dev = 0;
    if (cudaGetDevice(&dev) != cudaSuccess) return nullptr;
    std::lock_guard<std::mutex> lock(mu);
    auto it = pools.find(dev);
    if (it != pools.end()) return it->second;
    cudaMemPoolProps props = {};
    props.allocType = cudaMemAllocationTypePinned;
    props.location.type = cudaMemLocationTypeDevice;
    props.location.id = dev;
    cudaMemPool_t pool = nullptr;
    if (cudaMemPoolCreate(&pool, &props) != cudaSuccess) return nullptr;
    uint64_t keep = 8ull << 30;
    if (const char* v = getenv("FSGC_POOL_KEEP_BYTES")) keep = strtoull(v, nullptr, 10);
    cudaMemPoolSetAttribute(pool, cudaMemPoolAttrReleaseThreshold, &keep);
    pools[dev] = pool;
    return pool;
}

extern "C" int fsgc_load_graph(const void* edges, int64_t E, int ib, int64_t n, int on_device,
                               void* stream_, fsgc_graph** out) {
    if (!out) FSGC_FAIL(FSGC_ERR_INVALID, "fsgc_load_graph: out is NULL");
    *out = nullptr;
    if (E < 0 || (E > 0 && !edges)) FSGC_FAIL(FSGC_ERR_INVALID, "fsgc_load_graph: bad edge list");
    if (ib != 4 && ib != 8) FSGC_FAIL(FSGC_ERR_INVALID, "index_bytes must be 4 or 8");
    if (n <= 0 || n >= (1ll << 31)) FSGC_FAIL(FSGC_ERR_INVALID, "num_vertices must be in [1, 2^31)");
    cudaStream_t st = (cudaStream_t)stream_;
    int dev = 0;
    FSGC_CUDA(cudaGetDevice(&dev));
    if (!fsgc_device_pool()) FSGC_FAIL(FSGC_ERR_CUDA, "fsgc_load_graph: cannot create the memory pool");

    int B = 1;
    while ((1ll << B) < n) ++B;
    const int keybits = 2 * B;
    const uint64_t sentinel = (keybits == 64) ? ~0ull : ((1ull << keybits) - 1);

    // 1 emit
    DevBuf<char> din;
    const void* dedges = edges;
    if (!on_device && E > 0) {
        FSGC_CUDA(din.alloc((size_t)E * 2 * ib, st));
        FSGC_CUDA(cudaMemcpyAsync(din.ptr, edges, (size_t)E * 2 * ib, cudaMemcpyHostToDevice, st));
        dedges = din.ptr;
    }
    const int64_t K = 2 * E;
    DevBuf<uint64_t> ka, kb;
    DevBuf<int> dbad;
    FSGC_CUDA(ka.alloc(K > 0 ? K : 1, st));
    FSGC_CUDA(kb.alloc(K > 0 ? K : 1, st));
    FSGC_CUDA(dbad.alloc(1, st));
    FSGC_CUDA(cudaMemsetAsync(dbad.ptr, 0, sizeof(int), st));
    if (E > 0) {
        emit_keys<<<grid_for(E), 256, 0, st>>>(dedges, E, ib, n, B, sentinel, ka.ptr, dbad.ptr);
        FSGC_CUDA(cudaGetLastError());
    }
    din.release();

    // 2 sort, 3 unique
    DevBuf<char> tmp;
    size_t tmp_bytes = 0;
    DevBuf<int64_t> dnum;
    FSGC_CUDA(dnum.alloc(2, st));
    int64_t M = 0;
    if (K > 0) {
        cub::DoubleBuffer<uint64_t> db(ka.ptr, kb.ptr);
        FSGC_CUDA(cub::DeviceRadixSort::SortKeys(nullptr, tmp_bytes, db, K, 0, keybits, st));
        FSGC_CUDA(tmp.alloc(tmp_bytes, st));
        FSGC_CUDA(cub::DeviceRadixSort::SortKeys(tmp.ptr, tmp_bytes, db, K, 0, keybits, st));
        uint64_t* sorted = db.Current();
        uint64_t* other = db.Alternate();
        size_t ub = 0;
        FSGC_CUDA(cub::DeviceSelect::Unique(nullptr, ub, sorted, other, dnum.ptr, K, st));
        if (ub > tmp_bytes) { FSGC_CUDA(tmp.alloc(ub, st)); tmp_bytes = ub; }
        FSGC_CUDA(cub::DeviceSelect::Unique(tmp.ptr, ub, sorted, other, dnum.ptr, K, st));
        unique_count<<<1, 1, 0, st>>>(other, dnum.ptr, sentinel);   // drop the sentinel run
        FSGC_CUDA(cudaGetLastError());
        if (other != ka.ptr) std::swap(ka.ptr, kb.ptr);  // unique keys now in ka
    }
    int64_t hv[2] = {0, 0};   // M, bad flag: one host synchronisation
    FSGC_CUDA(cudaMemcpyAsync(&hv[0], dnum.ptr, sizeof(int64_t), cudaMemcpyDeviceToHost, st));
    FSGC_CUDA(cudaMemcpyAsync(&hv[1], dbad.ptr, sizeof(int), cudaMemcpyDeviceToHost, st));
    FSGC_CUDA(cudaStreamSynchronize(st));
    if (K > 0) M = hv[0];
    const int bad = (int)hv[1];
    if (bad) FSGC_FAIL(FSGC_ERR_INVALID, "edge list contains a vertex id outside [0, %lld)", (long long)n);
    // the counting kernels index oriented edges (int32) and CSR positions
    // (uint32) in 32 bits: 2m must stay below 2^32
    if (M / 2 >= (1ll << 31))
        FSGC_FAIL(FSGC_ERR_INVALID, "graph has %lld distinct edges; the limit is 2^31 - 1", (long long)(M / 2));
    kb.release();

    // 4 degrees of the original ids
    DevBuf<int64_t> offs_old;
    FSGC_CUDA(offs_old.alloc(n + 1, st));
    lower_bounds<<<grid_for(n + 1), 256, 0, st>>>(ka.ptr, M, n, B, offs_old.ptr);
    FSGC_CUDA(cudaGetLastError());

    // 5 degree order
    DevBuf<uint64_t> vk, vk2;
    FSGC_CUDA(vk.alloc(n, st));
    FSGC_CUDA(vk2.alloc(n, st));
    degree_keys<<<grid_for(n), 256, 0, st>>>(offs_old.ptr, n, B, vk.ptr);
    FSGC_CUDA(cudaGetLastError());
    {
        int degbits = 1;
        while ((1ll << degbits) <= M) ++degbits;
        int endbit = B + degbits;
        if (endbit > 64) endbit = 64;
        cub::DoubleBuffer<uint64_t> db(vk.ptr, vk2.ptr);
        size_t b = 0;
        FSGC_CUDA(cub::DeviceRadixSort::SortKeys(nullptr, b, db, n, 0, endbit, st));
        if (b > tmp_bytes) { FSGC_CUDA(tmp.alloc(b, st)); tmp_bytes = b; }
        FSGC_CUDA(cub::DeviceRadixSort::SortKeys(tmp.ptr, b, db, n, 0, endbit, st));
        if (db.Current() != vk.ptr) std::swap(vk.ptr, vk2.ptr);
    }
    offs_old.release();
    DevBuf<int32_t> order, rank;
    DevBuf<int64_t> offs;
    FSGC_CUDA(order.alloc(n, st));
    FSGC_CUDA(rank.alloc(n, st));
    FSGC_CUDA(offs.alloc(n + 1, st));
    ranks_from_order<<<grid_for(n), 256, 0, st>>>(vk.ptr, n, B, order.ptr, rank.ptr, offs.ptr);
    FSGC_CUDA(cudaGetLastError());
    vk.release();
    vk2.release();
    {   // offsets = exclusive scan of new-order degrees (in place, n+1 items)
        FSGC_CUDA(cudaMemsetAsync(offs.ptr + n, 0, sizeof(int64_t), st));
        size_t b = 0;
        FSGC_CUDA(cub::DeviceScan::ExclusiveSum(nullptr, b, offs.ptr, offs.ptr, n + 1, st));
        if (b > tmp_bytes) { FSGC_CUDA(tmp.alloc(b, st)); tmp_bytes = b; }
        FSGC_CUDA(cub::DeviceScan::ExclusiveSum(tmp.ptr, b, offs.ptr, offs.ptr, n + 1, st));
    }

    // 6 relabel + sort
    DevBuf<int32_t> adj, row, osrc, odst;
    int64_t m = M / 2;
    if (M > 0) {
        relabel_keys<<<grid_for(M), 256, 0, st>>>(ka.ptr, M, B, rank.ptr);
        FSGC_CUDA(cudaGetLastError());
        FSGC_CUDA(kb.alloc(M, st));
        cub::DoubleBuffer<uint64_t> db(ka.ptr, kb.ptr);
        size_t b = 0;
        FSGC_CUDA(cub::DeviceRadixSort::SortKeys(nullptr, b, db, M, 0, keybits, st));
        if (b > tmp_bytes) { FSGC_CUDA(tmp.alloc(b, st)); tmp_bytes = b; }
        FSGC_CUDA(cub::DeviceRadixSort::SortKeys(tmp.ptr, b, db, M, 0, keybits, st));
        uint64_t* sorted = db.Current();
        uint64_t* spare = db.Alternate();
        // 7 CSR arrays + oriented edges
        FSGC_CUDA(adj.alloc(M, st));
        FSGC_CUDA(row.alloc(M, st));
        split_keys<<<grid_for(M), 256, 0, st>>>(sorted, M, B, row.ptr, adj.ptr);
        FSGC_CUDA(cudaGetLastError());
        UpperTri pred{B, (1ull << B) - 1};
        size_t sb = 0;
        FSGC_CUDA(cub::DeviceSelect::If(nullptr, sb, sorted, spare, dnum.ptr, M, pred, st));
        if (sb > tmp_bytes) { FSGC_CUDA(tmp.alloc(sb, st)); tmp_bytes = sb; }
        FSGC_CUDA(cub::DeviceSelect::If(tmp.ptr, sb, sorted, spare, dnum.ptr, M, pred, st));
        FSGC_CUDA(osrc.alloc(m, st));
        FSGC_CUDA(odst.alloc(m, st));
        split_keys<<<grid_for(m), 256, 0, st>>>(spare, m, B, osrc.ptr, odst.ptr);
        FSGC_CUDA(cudaGetLastError());
    }
    // oriented view: split points + exclusive scan of out-degrees
    DevBuf<int64_t> split, oofs;
    FSGC_CUDA(split.alloc(n, st));
    FSGC_CUDA(oofs.alloc(n + 1, st));
    FSGC_CUDA(cudaMemsetAsync(oofs.ptr + n, 0, sizeof(int64_t), st));
    split_points<<<grid_for(n), 256, 0, st>>>(offs.ptr, adj.ptr, n, split.ptr, oofs.ptr);
    FSGC_CUDA(cudaGetLastError());
    {
        size_t b = 0;
        FSGC_CUDA(cub::DeviceScan::ExclusiveSum(nullptr, b, oofs.ptr, oofs.ptr, n + 1, st));
        if (b > tmp_bytes) { FSGC_CUDA(tmp.alloc(b, st)); tmp_bytes = b; }
        FSGC_CUDA(cub::DeviceScan::ExclusiveSum(tmp.ptr, b, oofs.ptr, oofs.ptr, n + 1, st));
    }
    // Triangle listing from the middle vertex (support pass and triangle-core
    // pass, count.cu): rev index + work units of the middles b, split at
    // out(b) = capw into warp-table units (SEG in-entries) and block-table
    // units (FSGC_SUP_CHUNK in-entries).  The merge-kernel work list (every
    // oriented edge in merge-length order) only where the merge kernel runs:
    // graphs below FSGC_SUP_HASH_MIN_M edges (launch-latency bound: the merge
    // kernel alone is fastest there) or FSGC_SUP_MERGE_ONLY (the independent
    // check of the hash kernels).
    DevBuf<int32_t> sorder, ssrc, sdst, rev;
    DevBuf<uint64_t> units, units_big;
    DevBuf<int64_t> ucnt, ucnt_big;
    FSGC_CUDA(cudaMemsetAsync(dnum.ptr, 0, 2 * sizeof(int64_t), st));
    int64_t hash_min_m = 1 << 20;
    if (const char* v = getenv("FSGC_SUP_HASH_MIN_M")) hash_min_m = atoll(v);
    const bool use_hash = m >= hash_min_m;
    const bool merge_list = !use_hash || (getenv("FSGC_SUP_MERGE_ONLY") && atoi(getenv("FSGC_SUP_MERGE_ONLY")));
    // FSGC_SUP_CAPW (tests): warp-table cap below the compiled 256, so small
    // graphs reach the block-table kernels
    int64_t capw = FSGC_SUP_CAPW;
    if (const char* v = getenv("FSGC_SUP_CAPW")) capw = std::max<int64_t>(1, std::min<int64_t>(atoll(v), FSGC_SUP_CAPW));
    if (m > 0) {
        {   // rev = oriented edge ids in (b, a) order = the in-entries' CSR order
            DevBuf<uint64_t> rk0, rk1;
            DevBuf<int32_t> rv1;
            FSGC_CUDA(rk0.alloc(m, st));
            FSGC_CUDA(rk1.alloc(m, st));
            FSGC_CUDA(rev.alloc(m, st));
            FSGC_CUDA(rv1.alloc(m, st));
            rev_keys<<<grid_for(m), 256, 0, st>>>(osrc.ptr, odst.ptr, m, B, rk0.ptr, rev.ptr);
            FSGC_CUDA(cudaGetLastError());
            cub::DoubleBuffer<uint64_t> dk(rk0.ptr, rk1.ptr);
            cub::DoubleBuffer<int32_t> dv(rev.ptr, rv1.ptr);
            size_t b = 0;
            FSGC_CUDA(cub::DeviceRadixSort::SortPairs(nullptr, b, dk, dv, m, 0, keybits, st));
            if (b > tmp_bytes) { FSGC_CUDA(tmp.alloc(b, st)); tmp_bytes = b; }
            FSGC_CUDA(cub::DeviceRadixSort::SortPairs(tmp.ptr, b, dk, dv, m, 0, keybits, st));
            if (dv.Current() != rev.ptr) std::swap(rev.ptr, rv1.ptr);
        }
        FSGC_CUDA(ucnt.alloc(n + 1, st));
        FSGC_CUDA(ucnt_big.alloc(n + 1, st));
        unit_counts<<<grid_for(n + 1), 256, 0, st>>>(offs.ptr, split.ptr, n, ucnt.ptr, ucnt_big.ptr, capw,
                                                     (unsigned long long*)dnum.ptr + 1);
        FSGC_CUDA(cudaGetLastError());
        size_t b = 0;
        FSGC_CUDA(cub::DeviceScan::ExclusiveSum(nullptr, b, ucnt.ptr, ucnt.ptr, n + 1, st));
        if (b > tmp_bytes) { FSGC_CUDA(tmp.alloc(b, st)); tmp_bytes = b; }
        FSGC_CUDA(cub::DeviceScan::ExclusiveSum(tmp.ptr, b, ucnt.ptr, ucnt.ptr, n + 1, st));
        FSGC_CUDA(cub::DeviceScan::ExclusiveSum(tmp.ptr, b, ucnt_big.ptr, ucnt_big.ptr, n + 1, st));
        FSGC_CUDA(units.alloc((size_t)n + (size_t)m / FSGC_SUP_SEG + 1, st));   // >= sum ceil(in/SEG)
        FSGC_CUDA(units_big.alloc((size_t)n + (size_t)m / FSGC_SUP_CHUNK + 1, st));
        unit_fill<<<grid_for(n), 256, 0, st>>>(ucnt.ptr, n, units.ptr);
        FSGC_CUDA(cudaGetLastError());
        unit_fill<<<grid_for(n), 256, 0, st>>>(ucnt_big.ptr, n, units_big.ptr);
        FSGC_CUDA(cudaGetLastError());
    }
    if (m > 0 && merge_list) {
        DevBuf<uint32_t> k0, k1;
        DevBuf<int32_t> i1;
        FSGC_CUDA(k0.alloc(m, st));
        FSGC_CUDA(k1.alloc(m, st));
        FSGC_CUDA(sorder.alloc(m, st));
        FSGC_CUDA(i1.alloc(m, st));
        support_work_keys<<<grid_for(m), 256, 0, st>>>(offs.ptr, split.ptr, osrc.ptr, odst.ptr, m, k0.ptr, sorder.ptr);
        FSGC_CUDA(cudaGetLastError());
        cub::DoubleBuffer<uint32_t> dk(k0.ptr, k1.ptr);
        cub::DoubleBuffer<int32_t> dv(sorder.ptr, i1.ptr);
        size_t b = 0;
        FSGC_CUDA(cub::DeviceRadixSort::SortPairs(nullptr, b, dk, dv, m, 0, 20, st));
        if (b > tmp_bytes) { FSGC_CUDA(tmp.alloc(b, st)); tmp_bytes = b; }
        FSGC_CUDA(cub::DeviceRadixSort::SortPairs(tmp.ptr, b, dk, dv, m, 0, 20, st));
        if (dv.Current() != sorder.ptr) std::swap(sorder.ptr, i1.ptr);
        FSGC_CUDA(ssrc.alloc(m, st));
        FSGC_CUDA(sdst.alloc(m, st));
        gather_uv<<<grid_for(m), 256, 0, st>>>(sorder.ptr, osrc.ptr, odst.ptr, m, ssrc.ptr, sdst.ptr);
        FSGC_CUDA(cudaGetLastError());
    }
    tmp.release();
    ka.release();
    kb.release();
    rank.release();

    // hub bitmaps within a memory budget (default min(4 GiB, 5% of device
    // memory); FSGC_HUB_BYTES overrides), only for degree >= kHubMinDeg
    int64_t hub_base = n, hub_words = (n + 31) / 32;
    int64_t maxdeg = 0;   // the last vertex has the largest degree
    int64_t nunits = 0, nunits_big = 0, maxout_big = 0;
    DevBuf<uint32_t> hubs;
    {
        size_t free_b = 0, total_b = 0;
        FSGC_CUDA(cudaMemGetInfo(&free_b, &total_b));
        int64_t budget = std::min<int64_t>(4ll << 30, (int64_t)(total_b / 20));
        if (const char* v = getenv("FSGC_HUB_BYTES")) budget = atoll(v);
        budget = std::min<int64_t>(budget, (int64_t)(free_b / 4));
        const int64_t per = hub_words * 4;
        int64_t max_hubs = per > 0 ? budget / per : 0;
        if (max_hubs > n) max_hubs = n;
        // first v in [n - max_hubs, n) with deg(v) >= kHubMinDeg (degrees are
        // ascending in the new ids), and the maximum degree: one synchronisation
        int64_t hv2[2] = {n, 0};
        if (m > 0) {   // unit counts and the largest block-table out-degree
            FSGC_CUDA(cudaMemcpyAsync(&nunits, ucnt.ptr + n, sizeof(int64_t), cudaMemcpyDeviceToHost, st));
            FSGC_CUDA(cudaMemcpyAsync(&nunits_big, ucnt_big.ptr + n, sizeof(int64_t), cudaMemcpyDeviceToHost, st));
            FSGC_CUDA(cudaMemcpyAsync(&maxout_big, dnum.ptr + 1, sizeof(int64_t), cudaMemcpyDeviceToHost, st));
        }
        if (n > 0) {
            DevBuf<int64_t> hs;
            FSGC_CUDA(hs.alloc(2, st));
            hub_search<<<1, 1, 0, st>>>(offs.ptr, n, n - std::max<int64_t>(0, std::min<int64_t>(max_hubs, n)),
                                        M > 0 ? 256 : (int64_t)1 << 62, hs.ptr);
            FSGC_CUDA(cudaGetLastError());
            FSGC_CUDA(cudaMemcpyAsync(hv2, hs.ptr, 2 * sizeof(int64_t), cudaMemcpyDeviceToHost, st));
            FSGC_CUDA(cudaStreamSynchronize(st));
        }
        if (max_hubs > 0 && M > 0) hub_base = hv2[0];
        maxdeg = hv2[1];
        if (hub_base < n) {
            FSGC_CUDA(hubs.alloc((size_t)(n - hub_base) * hub_words, st));
            FSGC_CUDA(cudaMemsetAsync(hubs.ptr, 0, (size_t)(n - hub_base) * hub_words * 4, st));
            hub_bitmaps<<<grid_for(M), 256, 0, st>>>(offs.ptr, adj.ptr, hub_base, n, hub_words, hubs.ptr);
            FSGC_CUDA(cudaGetLastError());
        }
    }
    FSGC_CUDA(cudaStreamSynchronize(st));

    fsgc_graph* g = new fsgc_graph;
    static std::atomic<uint64_t> next_uid{1};
    g->uid = next_uid.fetch_add(1);
    g->n = n;
    g->m = m;
    g->max_degree = maxdeg;
    g->offsets = offs.take();
    g->adj = adj.take();
    g->row = row.take();
    g->osrc = osrc.take();
    g->odst = odst.take();
    g->order = order.take();
    g->split = split.take();
    g->oofs = oofs.take();
    g->sorder = sorder.take();
    g->ssrc = ssrc.take();
    g->sdst = sdst.take();
    g->nsup_merge = merge_list ? m : 0;
    g->sup_hash = use_hash ? 1 : 0;
    g->sup_units = units.take();
    g->nsup_units = nunits;
    g->sup_units_big = units_big.take();
    g->nsup_units_big = nunits_big;
    g->sup_capw = (int32_t)capw;
    g->sup_maxout = maxout_big;
    g->rev = rev.take();
    g->hub_base = hub_base;
    g->hub_words = hub_words;
    g->hub_bits = hubs.take();
    g->device = dev;
    *out = g;
    return FSGC_OK;
}

extern "C" int fsgc_graph_get_info(const fsgc_graph* g, fsgc_graph_info* o) {
    if (!g || !o) FSGC_FAIL(FSGC_ERR_INVALID, "fsgc_graph_get_info: null argument");
    o->num_vertices = g->n;
    o->num_edges = g->m;
    o->max_degree = g->max_degree;
    o->offsets = g->offsets;
    o->adj = g->adj;
    o->row = g->row;
    o->osrc = g->osrc;
    o->odst = g->odst;
    o->order = g->order;
    return FSGC_OK;
}

extern "C" int fsgc_graph_download(const fsgc_graph* g, int64_t* offsets, int32_t* adj, int32_t* order) {
    if (!g) FSGC_FAIL(FSGC_ERR_INVALID, "fsgc_graph_download: null graph");
    if (offsets) FSGC_CUDA(cudaMemcpy(offsets, g->offsets, (g->n + 1) * sizeof(int64_t), cudaMemcpyDeviceToHost));
    if (adj && g->m > 0) FSGC_CUDA(cudaMemcpy(adj, g->adj, 2 * g->m * sizeof(int32_t), cudaMemcpyDeviceToHost));
    if (order) FSGC_CUDA(cudaMemcpy(order, g->order, g->n * sizeof(int32_t), cudaMemcpyDeviceToHost));
    return FSGC_OK;
}

extern "C" void fsgc_free_graph(fsgc_graph* g) {
    if (!g) return;
    cudaFree(g->offsets);
    cudaFree(g->adj);
    cudaFree(g->row);
    cudaFree(g->osrc);
    cudaFree(g->odst);
    cudaFree(g->order);
    cudaFree(g->split);
    cudaFree(g->oofs);
    cudaFree(g->sorder);
    cudaFree(g->ssrc);
    cudaFree(g->sdst);
    cudaFree(g->sup_units);
    cudaFree(g->sup_units_big);
    cudaFree(g->rev);
    cudaFree(g->hub_bits);
    delete g;
}
