// Integer front end of the TGOpt hot path on sm_100a: batch -> targets,
// DedupFilter (Alg. 2) in a thread-block cluster over distributed shared
// memory, CacheLookup / slot assignment / CacheStore index insert (Alg. 1
// l.7-10, 17; Alg. 3 with FIFO), NghLookup as a
// warp-cooperative 32-ary search in the T-CSR, and row-address resolution.
#include <cooperative_groups.h>

#include "tg_internal.cuh"

namespace cg = cooperative_groups;

namespace tg {

// ---------------------------------------------------------------- batch prep
__global__ void k_prep_edges(const int32_t* __restrict__ src, const int32_t* __restrict__ dst,
                             const uint32_t* __restrict__ ts, int64_t n_edges, int batch,
                             const int* __restrict__ bidx, Level out, int* n_out) {
  int64_t lo = bidx ? (int64_t)(*bidx) * batch : 0;
  int64_t rem = n_edges - lo;
  int B = (int)(rem < batch ? (rem < 0 ? 0 : rem) : batch);
  for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < B; i += gridDim.x * blockDim.x) {
    // src || dst, both at the edge time
    out.node[i] = src[lo + i];
    out.node[B + i] = dst[lo + i];
    uint32_t t = ts[lo + i];
    out.ts[i] = t;
    out.ts[B + i] = t;
  }
  if (blockIdx.x == 0 && threadIdx.x == 0) *n_out = 2 * B;
}

void launch_prep_edges(const int32_t* src, const int32_t* dst, const uint32_t* ts, int64_t n_edges,
                       int batch, const int* bidx, Level out, int* n_out_dev, cudaStream_t st) {
  int blocks = (batch + 255) / 256;
  k_prep_edges<<<blocks, 256, 0, st>>>(src, dst, ts, n_edges, batch, bidx, out, n_out_dev);
}

__global__ void k_prep_nodes(const int32_t* __restrict__ nodes, const uint32_t* __restrict__ ts, int n,
                             Level out, int* n_out) {
  for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) {
    out.node[i] = nodes[i];
    out.ts[i] = ts[i];
  }
  if (blockIdx.x == 0 && threadIdx.x == 0) *n_out = n;
}

void launch_prep_nodes(const int32_t* nodes, const uint32_t* ts, int n, Level out, int* n_out_dev,
                       cudaStream_t st) {
  int blocks = n > 0 ? (n + 255) / 256 : 1;
  k_prep_nodes<<<blocks, 256, 0, st>>>(nodes, ts, n, out, n_out_dev);
}

// -------------------------------------------------- ordered block scan helper
// Exclusive prefix of `v` over threads in index order; returns block total.
__device__ __forceinline__ int block_excl_scan(int v, int* s_warp, int& total) {
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5, nw = (blockDim.x + 31) >> 5;
  int x = v;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    int y = __shfl_up_sync(0xffffffffu, x, o);
    if (lane >= o) x += y;
  }
  if (lane == 31) s_warp[w] = x;
  __syncthreads();
  if (w == 0) {
    int s = lane < nw ? s_warp[lane] : 0;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      int y = __shfl_up_sync(0xffffffffu, s, o);
      if (lane >= o) s += y;
    }
    s_warp[lane] = s;
  }
  __syncthreads();
  total = s_warp[nw - 1];
  int excl = x - v + (w > 0 ? s_warp[w - 1] : 0);
  __syncthreads();
  return excl;
}

// -------------------------------------------------------------- DedupFilter
// Alg. 2 with a cluster-wide hash table in distributed shared
// memory: phase B inserts every (n, t) key and keeps the minimum position;
// phase C marks first occurrences, ranks them with an ordered scan across the
// cluster (first-occurrence order, R8) and phase D reads the inverse index.
__global__ void __launch_bounds__(kDedupThreads, 1)
k_dedup(Level in, const int* __restrict__ n_dev, Level uniq, int32_t* __restrict__ inv,
        int* __restrict__ nu_dev, long long* cnt_n, long long* cnt_u, int* err) {
  extern __shared__ __align__(16) unsigned char smem[];
  unsigned long long* skey = reinterpret_cast<unsigned long long*>(smem);
  unsigned int* spos = reinterpret_cast<unsigned int*>(skey + kDedupSlots);
  __shared__ int s_warp[32];
  __shared__ int s_total;
  cg::cluster_group cluster = cg::this_cluster();
  const unsigned CL = cluster.num_blocks();
  const unsigned rank = cluster.block_rank();
  const int tid = threadIdx.x;
  const int n = *n_dev;
  for (int s = tid; s < kDedupSlots; s += blockDim.x) {
    skey[s] = kEmptyKey;
    spos[s] = 0xFFFFFFFFu;
  }
  cluster.sync();
  const int chunk = (n + (int)CL - 1) / (int)CL;
  const int cbeg = min(n, (int)rank * chunk), cend = min(n, cbeg + chunk);
  const int ipt = (chunk + (int)blockDim.x - 1) / (int)blockDim.x;
  const int tbeg = cbeg + tid * ipt;
  const unsigned long long tmask = (unsigned long long)CL * kDedupSlots - 1ull;
  unsigned slot[kDedupIPT];
  // ---- phase B: insert keys, keep the minimum position
#pragma unroll
  for (int j = 0; j < kDedupIPT; ++j) {
    slot[j] = 0xFFFFFFFFu;
    const int i = tbeg + j;
    if (j < ipt && i < cend) {
      const unsigned long long key = tkey(in.node[i], in.ts[i]);
      unsigned long long h = mix64(key) & tmask;
      for (unsigned long long probe = 0; probe <= tmask; ++probe) {
        const unsigned owner = (unsigned)(h / kDedupSlots), loc = (unsigned)(h % kDedupSlots);
        unsigned long long* kp = cluster.map_shared_rank(skey, owner) + loc;
        const unsigned long long old = atomicCAS(kp, kEmptyKey, key);
        if (old == kEmptyKey || old == key) {
          atomicMin(cluster.map_shared_rank(spos, owner) + loc, (unsigned)i);
          slot[j] = (unsigned)h;
          break;
        }
        h = (h + 1) & tmask;
      }
      if (slot[j] == 0xFFFFFFFFu) atomicOr(err, kErrDedupFull);
    }
  }
  cluster.sync();
  // ---- phase C1: first occurrences, ordered scan inside the CTA
  int cnt = 0;
  unsigned firstmask = 0;
#pragma unroll
  for (int j = 0; j < kDedupIPT; ++j) {
    const int i = tbeg + j;
    if (j < ipt && i < cend && slot[j] != 0xFFFFFFFFu) {
      const unsigned h = slot[j];
      const unsigned p = *(cluster.map_shared_rank(spos, h / kDedupSlots) + (h % kDedupSlots));
      if (p == (unsigned)i) {
        firstmask |= 1u << j;
        ++cnt;
      }
    }
  }
  int total;
  const int excl = block_excl_scan(cnt, s_warp, total);
  if (tid == 0) s_total = total;
  cluster.sync();  // all first-decisions done; CTA totals visible
  int base = 0;
  for (unsigned r = 0; r < rank; ++r) base += *cluster.map_shared_rank(&s_total, r);
  // ---- phase C2: unique list in first-occurrence order; slot -> unique id
  int uid = base + excl;
#pragma unroll
  for (int j = 0; j < kDedupIPT; ++j) {
    if (firstmask & (1u << j)) {
      const int i = tbeg + j;
      uniq.node[uid] = in.node[i];
      uniq.ts[uid] = in.ts[i];
      const unsigned h = slot[j];
      *(cluster.map_shared_rank(spos, h / kDedupSlots) + (h % kDedupSlots)) = (unsigned)uid;
      ++uid;
    }
  }
  if (rank == CL - 1 && tid == 0) {
    const int u = base + s_total;
    *nu_dev = u;
    if (cnt_n) atomicAdd((unsigned long long*)cnt_n, (unsigned long long)n);
    if (cnt_u) atomicAdd((unsigned long long*)cnt_u, (unsigned long long)u);
  }
  cluster.sync();
  // ---- phase D: inverse index (DedupInvert map, Alg. 1 l.20)
#pragma unroll
  for (int j = 0; j < kDedupIPT; ++j) {
    const int i = tbeg + j;
    if (j < ipt && i < cend && slot[j] != 0xFFFFFFFFu) {
      const unsigned h = slot[j];
      inv[i] = (int32_t) * (cluster.map_shared_rank(spos, h / kDedupSlots) + (h % kDedupSlots));
    }
  }
  cluster.sync();  // peers may still read this CTA's shared memory
}

// dedup disabled (ablation): identity unique list and inverse index
__global__ void k_dedup_off(Level in, const int* __restrict__ n_dev, Level uniq, int32_t* __restrict__ inv,
                            int* __restrict__ nu_dev, long long* cnt_n, long long* cnt_u) {
  const int n = *n_dev;
  for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) {
    uniq.node[i] = in.node[i];
    uniq.ts[i] = in.ts[i];
    inv[i] = i;
  }
  if (blockIdx.x == 0 && threadIdx.x == 0) {
    *nu_dev = n;
    if (cnt_n) atomicAdd((unsigned long long*)cnt_n, (unsigned long long)n);
    if (cnt_u) atomicAdd((unsigned long long*)cnt_u, (unsigned long long)n);
  }
}

static int dedup_cluster_size(int n_max) {
  int cl = 1;
  while (cl < 16 && (long long)cl * 10000 < n_max) cl <<= 1;
  return cl;
}

void launch_dedup(Level in, const int* n_dev, int n_max, Level uniq, int32_t* inv, int* nu_dev,
                  long long* cnt_n, long long* cnt_u, bool dedup_on, int* err, cudaStream_t st) {
  if (!dedup_on) {
    int blocks = (n_max + 255) / 256;
    if (blocks < 1) blocks = 1;
    if (blocks > 1184) blocks = 1184;
    k_dedup_off<<<blocks, 256, 0, st>>>(in, n_dev, uniq, inv, nu_dev, cnt_n, cnt_u);
    return;
  }
  const int cl = dedup_cluster_size(n_max);
  const size_t smem = (size_t)kDedupSlots * (sizeof(unsigned long long) + sizeof(unsigned));
  static bool attr_done = false;
  if (!attr_done) {
    cudaFuncSetAttribute(k_dedup, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    cudaFuncSetAttribute(k_dedup, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
    attr_done = true;
  }
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(cl);
  cfg.blockDim = dim3(kDedupThreads);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = st;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeClusterDimension;
  attr[0].val.clusterDim.x = cl;
  attr[0].val.clusterDim.y = 1;
  attr[0].val.clusterDim.z = 1;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  cudaLaunchKernelEx(&cfg, k_dedup, in, n_dev, uniq, inv, nu_dev, cnt_n, cnt_u, err);
}

// ------------------------------------------------------- CacheLookup / Store
// One CTA: probe every unique key of layer l (Alg. 1 l.7-8), rank the misses
// in unique-list order (l.10: "shrink ... to only the misses"), give each miss
// the next FIFO ring position and insert key -> position into the index
// (CacheStore, Alg. 3). Eviction is logical: the live window is the newest
// `limit` positions (R11); dead index entries are reclaimed by later inserts.
__device__ __forceinline__ unsigned long long ld_volatile_u64(const unsigned long long* p) {
  return *(const volatile unsigned long long*)p;
}

__global__ void __launch_bounds__(1024, 1)
k_probe(Level uniq, const int* __restrict__ nu_dev, CacheDev c, int cache_on, int32_t* __restrict__ c_uidx,
        Level C, int* __restrict__ nc_dev, long long* __restrict__ slot, long long* cntl, int* err) {
  __shared__ int s_warp[32];
  const int n = *nu_dev;
  const long long head = c.state[0], size = c.state[1], limit = c.state[2];
  const long long live_lo = head - size;
  const int tid = threadIdx.x;
  const int ipt = (n + (int)blockDim.x - 1) / (int)blockDim.x;
  const int tbeg = tid * ipt;
  int cnt = 0;
  unsigned missmask = 0;
  // ---- probe (no inserts happen until every probe is done)
#pragma unroll
  for (int j = 0; j < kDedupIPT; ++j) {
    const int i = tbeg + j;
    if (j < ipt && i < n) {
      bool hit = false;
      long long hp = 0;
      if (cache_on) {
        const unsigned long long key = tkey(uniq.node[i], uniq.ts[i]);
        unsigned long long h = mix64(key) & c.imask;
        for (unsigned long long pr = 0; pr <= c.imask; ++pr) {
          const unsigned long long k0 = c.ikey[h];
          if (k0 == kEmptyKey) break;
          if (k0 == key) {
            const long long p = c.ipos[h];
            if (p >= live_lo) {
              hit = true;
              hp = p;
              break;
            }
          }
          h = (h + 1) & c.imask;
        }
      }
      if (hit) {
        slot[i] = hp % c.rcap;
      } else {
        missmask |= 1u << j;
        ++cnt;
      }
    }
  }
  int m;
  const int excl = block_excl_scan(cnt, s_warp, m);
  // ---- misses: ring position, miss list, index insert
  int r = excl;
#pragma unroll
  for (int j = 0; j < kDedupIPT; ++j) {
    if (missmask & (1u << j)) {
      const int i = tbeg + j;
      const long long pos = head + r;
      slot[i] = pos % c.rcap;
      c_uidx[r] = i;
      C.node[r] = uniq.node[i];
      C.ts[r] = uniq.ts[i];
      if (cache_on) {
        const unsigned long long key = tkey(uniq.node[i], uniq.ts[i]);
        unsigned long long h = mix64(key) & c.imask;
        bool done = false;
        for (unsigned long long pr = 0; pr <= 4 * c.imask && !done; ++pr) {
          const unsigned long long k0 = ld_volatile_u64(c.ikey + h);
          if (k0 != kLockedKey) {
            __threadfence();
            const bool reusable =
                (k0 == kEmptyKey) || (k0 == key) || (*(volatile long long*)(c.ipos + h) < live_lo);
            if (reusable) {
              if (atomicCAS(c.ikey + h, k0, kLockedKey) == k0) {
                *(volatile long long*)(c.ipos + h) = pos;
                __threadfence();
                atomicExch(c.ikey + h, key);
                if (k0 == kEmptyKey) atomicAdd((unsigned long long*)(c.state + 3), 1ull);
                done = true;
              }
              continue;  // lost the race: re-read the same slot
            }
          }
          h = (h + 1) & c.imask;
        }
        if (!done) atomicOr(err, kErrIndexFull);
      }
      ++r;
    }
  }
  __syncthreads();
  if (tid == 0) {
    *nc_dev = m;
    if (cache_on) {
      const long long nsz = size + m < limit ? size + m : limit;
      const long long ev_total = size + m - nsz;
      const long long evicted = ev_total < size ? ev_total : size;
      c.state[0] = head + m;
      c.state[1] = nsz;
      if (cntl) {
        atomicAdd((unsigned long long*)(cntl + 2), (unsigned long long)n);      // lookups
        atomicAdd((unsigned long long*)(cntl + 3), (unsigned long long)(n - m));  // hits
        atomicAdd((unsigned long long*)(cntl + 4), (unsigned long long)m);      // misses
        atomicAdd((unsigned long long*)(cntl + 5), (unsigned long long)evicted);
      }
      if (c.state[3] * 10 > (long long)(c.imask + 1) * 9) atomicOr(err, kErrIndexFull);
    } else {
      c.state[0] = head + m;  // ring used as per-batch scratch
      if (cntl) atomicAdd((unsigned long long*)(cntl + 4), (unsigned long long)m);
    }
  }
}

void launch_probe(Level uniq, const int* nu_dev, int nu_max, CacheDev cache, bool cache_on, int32_t* c_uidx,
                  Level C, int* nc_dev, long long* slot, long long* cnt_layer, int* err, cudaStream_t st) {
  (void)nu_max;  // <= 1024 * kDedupIPT, checked by the host
  k_probe<<<1, 1024, 0, st>>>(uniq, nu_dev, cache, cache_on ? 1 : 0, c_uidx, C, nc_dev, slot, cnt_layer, err);
}

// Top layer: C_L = U_L (no lookup at l = L, R9).
__global__ void k_copy_level(Level in, const int* __restrict__ n_dev, Level out, int32_t* __restrict__ c_uidx,
                             int* __restrict__ n_out, long long* cnt_miss) {
  const int n = *n_dev;
  for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) {
    out.node[i] = in.node[i];
    out.ts[i] = in.ts[i];
    c_uidx[i] = i;
  }
  if (blockIdx.x == 0 && threadIdx.x == 0) {
    *n_out = n;
    if (cnt_miss) atomicAdd((unsigned long long*)cnt_miss, (unsigned long long)n);
  }
}

void launch_copy_level(Level in, const int* n_dev, int n_max, Level out, int32_t* c_uidx, int* n_out_dev,
                       long long* cnt_miss, cudaStream_t st) {
  int blocks = (n_max + 255) / 256;
  if (blocks < 1) blocks = 1;
  k_copy_level<<<blocks, 256, 0, st>>>(in, n_dev, out, c_uidx, n_out_dev, cnt_miss);
}

// ------------------------------------------------------------------ NghLookup
// Warp per target: 32-ary search for the first adjacency entry with t_j >= t
// (strict t_j < t), then lanes copy the last min(k, p-lo) entries
// right-aligned (R6), padding (0, 0, 0) on the left (R7).
__global__ void k_sample(GraphDev g, Level C, const int* __restrict__ nc_dev, int k, Level next,
                         int32_t* __restrict__ eid, int* __restrict__ n_next, int* err) {
  const int nC = *nc_dev;
  const int lane = threadIdx.x & 31;
  const int warp = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int nwarps = (gridDim.x * blockDim.x) >> 5;
  if (warp == 0 && lane == 0) *n_next = nC * (k + 1);
  for (int p = warp; p < nC; p += nwarps) {
    int i = C.node[p];
    const uint32_t t = C.ts[p];
    if (i < 0 || i > g.V) {
      if (lane == 0) atomicOr(err, kErrNodeRange);
      i = 0;
    }
    int a = g.rowptr[i], b = g.rowptr[i + 1];
    // invariant: the first entry with t_j >= t lies in [a, b] (b = "none")
    while (b - a > 31) {
      const int step = (b - a + 31) >> 5;
      const int x = a + lane * step;
      const bool ge = (x < b) ? (g.adj_t[x] >= t) : true;
      const unsigned msk = __ballot_sync(0xffffffffu, ge);
      if (msk == 0) {  // every probe is < t: answer beyond the last probe
        a = a + 31 * step + 1;
        continue;
      }
      const int f = __ffs(msk) - 1;
      const int nb = a + f * step;
      a = (f == 0) ? a : a + (f - 1) * step + 1;
      b = nb < b ? nb : b;
    }
    {
      // b - a <= 31: lane (b - a) probes x == b and votes true, so msk != 0
      const int x = a + lane;
      const bool ge = (x < b) ? (g.adj_t[x] >= t) : true;
      const unsigned msk = __ballot_sync(0xffffffffu, ge);
      a = a + (__ffs(msk) - 1);
    }
    const int lo = g.rowptr[i];
    const int cnt = min(k, a - lo);
    if (lane < k) {
      int nb = 0, e = 0;
      uint32_t tj = 0;
      if (lane >= k - cnt) {
        const int x = a - k + lane;
        nb = g.adj_nbr[x];
        e = g.adj_eid[x];
        tj = g.adj_t[x];
      }
      next.node[nC + p * k + lane] = nb;
      next.ts[nC + p * k + lane] = tj;
      eid[p * k + lane] = e;
    }
    if (lane == 0) {
      next.node[p] = C.node[p];
      next.ts[p] = t;
    }
  }
}

void launch_sample(const GraphDev& g, Level C, const int* nc_dev, int nc_max, int k, Level next, int32_t* eid,
                   int* n_next_dev, int* err, cudaStream_t st) {
  int blocks = (nc_max * 32 + 255) / 256;
  if (blocks < 1) blocks = 1;
  if (blocks > 148 * 8) blocks = 148 * 8;
  k_sample<<<blocks, 256, 0, st>>>(g, C, nc_dev, k, next, eid, n_next_dev, err);
}

// ---------------------------------------------------------------- row lookup
__global__ void k_resolve(const float* __restrict__ X, int ldn, int64_t V, int lm1_is_zero, Level prev,
                          const int* __restrict__ nprev_dev, const int32_t* __restrict__ inv_prev,
                          const long long* __restrict__ slot_prev, const float* __restrict__ ring_prev,
                          const int* __restrict__ nc_dev, const int32_t* __restrict__ c_uidx,
                          const long long* __restrict__ slot_cur, float* ring_cur, float* hl_out,
                          const float** __restrict__ rows, float** __restrict__ dst, int* err) {
  const int np = *nprev_dev, nC = *nc_dev;
  const int tid = blockIdx.x * blockDim.x + threadIdx.x, nt = gridDim.x * blockDim.x;
  for (int j = tid; j < np; j += nt) {
    const float* r;
    if (lm1_is_zero) {
      int node = prev.node[j];
      if (node < 0 || node > V) {
        atomicOr(err, kErrNodeRange);
        node = 0;
      }
      r = X + (size_t)node * ldn;  // h^(0) = x_i (Alg. 1 l.2-3)
    } else {
      r = ring_prev + (size_t)slot_prev[inv_prev[j]] * ldn;  // H^(l-1) via inv (l.20)
    }
    rows[j] = r;
  }
  for (int p = tid; p < nC; p += nt)
    dst[p] = ring_cur ? ring_cur + (size_t)slot_cur[c_uidx[p]] * ldn : hl_out + (size_t)p * ldn;
}

void launch_resolve(const GraphDev& g, int lm1_is_zero, Level prev, const int* nprev_dev, int nprev_max,
                    const int32_t* inv_prev, const long long* slot_prev, const float* ring_prev,
                    long long rcap_prev, int ld, const int* nc_dev, int nc_max, const int32_t* c_uidx,
                    const long long* slot_cur, float* ring_cur, long long rcap_cur, float* hl_out,
                    const float** rows, float** dst, int* err, cudaStream_t st) {
  (void)rcap_prev;
  (void)rcap_cur;
  (void)ld;
  int mx = nprev_max > nc_max ? nprev_max : nc_max;
  int blocks = (mx + 255) / 256;
  if (blocks < 1) blocks = 1;
  if (blocks > 592) blocks = 592;
  k_resolve<<<blocks, 256, 0, st>>>(g.X, g.ldn, g.V, lm1_is_zero, prev, nprev_dev, inv_prev, slot_prev,
                                    ring_prev, nc_dev, c_uidx, slot_cur, ring_cur, hl_out, rows, dst, err);
}

// ------------------------------------------------------------------- misc
__global__ void k_bump(int* b) { *b += 1; }
void launch_bump(int* bidx, cudaStream_t st) { k_bump<<<1, 1, 0, st>>>(bidx); }

__global__ void k_add_counters(const long long* __restrict__ src, long long* __restrict__ dst, int n) {
  int i = threadIdx.x;
  if (i < n) dst[i] += src[i];
}
void launch_add_counters(const long long* src, long long* dst, int n, cudaStream_t st) {
  k_add_counters<<<1, 128, 0, st>>>(src, dst, n);
}

}  // namespace tg
