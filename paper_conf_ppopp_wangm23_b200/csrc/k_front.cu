// Integer front end of the TGOpt hot path on sm_100a, per superbatch:
//  * DedupFilter (Alg. 2): one thread-block cluster per batch, the
//    hash table lives in the cluster's distributed shared memory;
//  * CacheLookup / compaction / CacheStore index insert (Alg. 1 l.7-10, l.17;
//    Alg. 3 with the FIFO limit of P:L330-332), batch after batch in one CTA so
//    the per-batch cache semantics are exactly the sequential ones;
//  * NghLookup: warp per target, 32-ary search in the T-CSR;
//  * row-address resolution for the dense stages.
#include <cooperative_groups.h>

#include "tg_internal.cuh"

namespace cg = cooperative_groups;

namespace tg {

// -------------------------------------------------- ordered block scan helper
// Exclusive prefix of `v` over threads in index order; total via `total`.
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

__device__ __forceinline__ int batch_edges(const EdgeSrc& es, int b, int64_t& lo) {
  lo = es.e0 + (int64_t)b * es.B;
  const int64_t rem = es.n_edges - lo;
  return (int)(rem < es.B ? (rem < 0 ? 0 : rem) : es.B);
}

// -------------------------------------------------------------- DedupFilter
// Phase B inserts every (n, t) key into the cluster-wide table (DSMEM) and
// keeps the minimum position; phase C marks first occurrences and ranks them
// with an ordered scan across the cluster (first-occurrence order, R8);
// phase D reads the inverse index.
__global__ void __launch_bounds__(kDedupThreads, 1)
k_dedup(LevelDev lv, int edge_mode, EdgeSrc es, long long* cnt, int layer, int* err, int nslots) {
  // nslots: hash slots per CTA (power of two, sized to the batch: load <= 0.4)
  extern __shared__ __align__(16) unsigned char smem[];
  unsigned long long* skey = reinterpret_cast<unsigned long long*>(smem);
  unsigned int* spos = reinterpret_cast<unsigned int*>(skey + nslots);
  __shared__ int s_warp[32];
  __shared__ int s_total;
  cg::cluster_group cluster = cg::this_cluster();
  const unsigned CL = cluster.num_blocks();
  const unsigned rank = cluster.block_rank();
  const int b = blockIdx.x / CL;
  const int tid = threadIdx.x;
  int64_t elo = 0;
  int Bb = 0, n;
  if (edge_mode) {
    Bb = batch_edges(es, b, elo);
    n = (es.neg ? 3 : 2) * Bb;  // targets src || dst (|| neg) at the edge time
  } else {
    n = lv.n_in[b];
  }
  const size_t seg = (size_t)b * lv.cap;
  auto item = [&](int i, int32_t& node, uint32_t& t) {
    if (edge_mode) {
      const int part = i < Bb ? 0 : (i < 2 * Bb ? 1 : 2);
      const int64_t e = elo + (i - part * Bb);
      node = part == 0 ? es.src[e] : (part == 1 ? es.dst[e] : es.neg[e]);
      t = es.ts[e];
    } else {
      node = lv.in_node[seg + i];
      t = lv.in_ts[seg + i];
    }
  };
  for (int s = tid; s < nslots; s += blockDim.x) {
    skey[s] = kEmptyKey;
    spos[s] = 0xFFFFFFFFu;
  }
  pdl_enter();  // shared-memory setup above overlaps the previous kernel's tail
  cluster.sync();
  const int chunk = (n + (int)CL - 1) / (int)CL;
  const int cbeg = min(n, (int)rank * chunk), cend = min(n, cbeg + chunk);
  const int ipt = (chunk + (int)blockDim.x - 1) / (int)blockDim.x;
  const int tbeg = cbeg + tid * ipt;
  const unsigned long long tmask = (unsigned long long)CL * nslots - 1ull;
  unsigned slot[kDedupIPT];
  // ---- phase B
#pragma unroll
  for (int j = 0; j < kDedupIPT; ++j) {
    slot[j] = 0xFFFFFFFFu;
    const int i = tbeg + j;
    if (j < ipt && i < cend) {
      int32_t node;
      uint32_t t;
      item(i, node, t);
      const unsigned long long key = tkey(node, t);
      unsigned long long h = mix64(key) & tmask;
      for (unsigned long long probe = 0; probe <= tmask; ++probe) {
        const unsigned owner = (unsigned)(h / nslots), loc = (unsigned)(h % nslots);
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
  // ---- phase C1: first occurrences
  int c = 0;
  unsigned firstmask = 0;
#pragma unroll
  for (int j = 0; j < kDedupIPT; ++j) {
    const int i = tbeg + j;
    if (j < ipt && i < cend && slot[j] != 0xFFFFFFFFu) {
      const unsigned h = slot[j];
      const unsigned p = *(cluster.map_shared_rank(spos, h / nslots) + (h % nslots));
      if (p == (unsigned)i) {
        firstmask |= 1u << j;
        ++c;
      }
    }
  }
  int total;
  const int excl = block_excl_scan(c, s_warp, total);
  if (tid == 0) s_total = total;
  cluster.sync();
  int base = 0;
  for (unsigned r = 0; r < rank; ++r) base += *cluster.map_shared_rank(&s_total, r);
  // ---- phase C2: unique list in first-occurrence order; slot -> unique id
  int uid = base + excl;
#pragma unroll
  for (int j = 0; j < kDedupIPT; ++j) {
    if (firstmask & (1u << j)) {
      const int i = tbeg + j;
      int32_t node;
      uint32_t t;
      item(i, node, t);
      lv.u_node[seg + uid] = node;
      lv.u_ts[seg + uid] = t;
      const unsigned h = slot[j];
      *(cluster.map_shared_rank(spos, h / nslots) + (h % nslots)) = (unsigned)uid;
      ++uid;
    }
  }
  if (rank == CL - 1 && tid == 0) {
    const int u = base + s_total;
    lv.n_u[b] = u;
    if (edge_mode) lv.n_in[b] = n;
    cnt_add(cnt, b, layer * TG_CNT_PER_LAYER + 0, n);
    cnt_add(cnt, b, layer * TG_CNT_PER_LAYER + 1, u);
  }
  cluster.sync();
  // ---- phase D: inverse index (DedupInvert map, Alg. 1 l.20)
#pragma unroll
  for (int j = 0; j < kDedupIPT; ++j) {
    const int i = tbeg + j;
    if (j < ipt && i < cend && slot[j] != 0xFFFFFFFFu) {
      const unsigned h = slot[j];
      lv.inv[seg + i] = (int32_t) * (cluster.map_shared_rank(spos, h / nslots) + (h % nslots));
    }
  }
  cluster.sync();  // peers may still read this CTA's shared memory
}

// dedup disabled (ablation): identity unique list and inverse index
__global__ void k_dedup_off(LevelDev lv, int S, int edge_mode, EdgeSrc es, long long* cnt, int layer) { pdl_enter();
  for (int b = blockIdx.y; b < S; b += gridDim.y) {
    int64_t elo = 0;
    int Bb = 0, n;
    if (edge_mode) {
      Bb = batch_edges(es, b, elo);
      n = (es.neg ? 3 : 2) * Bb;
    } else {
      n = lv.n_in[b];
    }
    const size_t seg = (size_t)b * lv.cap;
    for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) {
      int32_t node;
      uint32_t t;
      if (edge_mode) {
        const int part = i < Bb ? 0 : (i < 2 * Bb ? 1 : 2);
        const int64_t e = elo + (i - part * Bb);
        node = part == 0 ? es.src[e] : (part == 1 ? es.dst[e] : es.neg[e]);
        t = es.ts[e];
      } else {
        node = lv.in_node[seg + i];
        t = lv.in_ts[seg + i];
      }
      lv.u_node[seg + i] = node;
      lv.u_ts[seg + i] = t;
      lv.inv[seg + i] = i;
    }
    if (blockIdx.x == 0 && threadIdx.x == 0) {
      lv.n_u[b] = n;
      if (edge_mode) lv.n_in[b] = n;
      cnt_add(cnt, b, layer * TG_CNT_PER_LAYER + 0, n);
      cnt_add(cnt, b, layer * TG_CNT_PER_LAYER + 1, n);
    }
  }
}

static int dedup_cluster_size(int n_max) {
  int cl = 1;
  // ~2.5k items per CTA: enough threads per batch that the phases are short
  while (cl < 16 && ((long long)cl * 2560 < n_max || (long long)cl * 10000 < n_max)) cl <<= 1;
  return cl;
}

void launch_dedup(LevelDev lv, int S, int n_max, bool edge_mode, EdgeSrc es, long long* cnt, int layer,
                  bool dedup_on, int* err, cudaStream_t st) {
  if (!dedup_on) {
    int bx = (n_max + 255) / 256;
    if (bx < 1) bx = 1;
    if (bx > 64) bx = 64;
    launch_k(k_dedup_off, dim3(dim3(bx, S)), dim3(256), 0, st, lv, S, edge_mode ? 1 : 0, es, cnt, layer);
    return;
  }
  const int cl = dedup_cluster_size(n_max);
  int nslots = 1024;  // per CTA: cl * nslots >= 2.5 n_max (load <= 0.4)
  while (nslots < kDedupSlots && (long long)cl * nslots * 2 < (long long)n_max * 5) nslots <<= 1;
  const size_t smem = (size_t)nslots * (sizeof(unsigned long long) + sizeof(unsigned));
  static bool attr_done = false;
  if (!attr_done) {
    cudaFuncSetAttribute(k_dedup, cudaFuncAttributeMaxDynamicSharedMemorySize,
                         (int)((size_t)kDedupSlots * (sizeof(unsigned long long) + sizeof(unsigned))));
    cudaFuncSetAttribute(k_dedup, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
    attr_done = true;
  }
  launch_k_cluster(k_dedup, dim3(cl * S), dim3(kDedupThreads), smem, st, cl, lv, edge_mode ? 1 : 0, es, cnt, layer,
                   err, nslots);
}

// ------------------------------------------------------- CacheLookup / Store
// One CTA walks the S batches in order. For each batch: probe every unique
// key (Alg. 1 l.7-8), rank the misses in unique-list order (l.10), append them
// to the compute list, give each miss the next FIFO ring position and insert
// key -> position into the index (CacheStore, Alg. 3). Eviction is logical:
// the live window is the newest `limit` positions (R11); dead index entries
// are reclaimed by later inserts. The next batch probes only after this
// batch's inserts (bar.sync orders the CTA's global writes).
__device__ __forceinline__ unsigned long long ld_volatile_u64(const unsigned long long* p) {
  return *(const volatile unsigned long long*)p;
}

__global__ void __launch_bounds__(1024, 1)
k_probe(LevelDev lv, int S, CacheDev c, int use_cache, int has_ring, long long* cnt, int layer, int* err) { pdl_enter();
  __shared__ int s_warp[32];
  __shared__ int s_base;
  __shared__ long long s_head, s_size;
  const int tid = threadIdx.x;
  if (tid == 0) {
    s_base = 0;
    s_head = has_ring ? c.state[0] : 0;
    s_size = has_ring ? c.state[1] : 0;
  }
  const long long limit = has_ring ? c.state[2] : 0;
  for (int b = 0; b < S; ++b) {
    __syncthreads();
    const int n = lv.n_u[b];
    const long long head = s_head, size = s_size;
    const long long live_lo = head - size;
    const int base = s_base;
    const size_t seg = (size_t)b * lv.cap;
    const int ipt = (n + (int)blockDim.x - 1) / (int)blockDim.x;
    const int tbeg = tid * ipt;
    int m_local = 0;
    unsigned missmask = 0;
#pragma unroll
    for (int j = 0; j < kProbeIPT; ++j) {
      const int i = tbeg + j;
      if (j < ipt && i < n) {
        bool hit = false;
        long long hp = 0;
        if (use_cache) {
          const unsigned long long key = tkey(lv.u_node[seg + i], lv.u_ts[seg + i]);
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
          lv.slot[seg + i] = hp % c.rcap;
        } else {
          missmask |= 1u << j;
          ++m_local;
        }
      }
    }
    int m;
    const int excl = block_excl_scan(m_local, s_warp, m);
    int r = excl;
#pragma unroll
    for (int j = 0; j < kProbeIPT; ++j) {
      if (missmask & (1u << j)) {
        const int i = tbeg + j;
        const int q = base + r;
        const int32_t node = lv.u_node[seg + i];
        const uint32_t t = lv.u_ts[seg + i];
        lv.c_b[q] = b;
        lv.c_u[q] = i;
        lv.c_node[q] = node;
        lv.c_ts[q] = t;
        if (has_ring) {
          const long long pos = head + r;
          lv.slot[seg + i] = pos % c.rcap;
          if (use_cache) {
            const unsigned long long key = tkey(node, t);
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
                    __threadfence();  // re-check under the lock (ABA, see k_probe_ins)
                    if (k0 != kEmptyKey && k0 != key && *(volatile long long*)(c.ipos + h) >= live_lo) {
                      atomicExch(c.ikey + h, k0);
                      h = (h + 1) & c.imask;
                      continue;
                    }
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
        }
        ++r;
      }
    }
    __syncthreads();
    if (tid == 0) {
      lv.c_base[b] = base;
      lv.n_c[b] = m;
      s_base = base + m;
      const int L6 = layer * TG_CNT_PER_LAYER;
      if (use_cache) {
        const long long nsz = size + m < limit ? size + m : limit;
        const long long ev_total = size + m - nsz;
        const long long evicted = ev_total < size ? ev_total : size;
        s_head = head + m;
        s_size = nsz;
        cnt_add(cnt, b, L6 + 2, n);      // lookups
        cnt_add(cnt, b, L6 + 3, n - m);  // hits
        cnt_add(cnt, b, L6 + 4, m);      // misses = embeddings computed
        cnt_add(cnt, b, L6 + 5, evicted);
      } else {
        if (has_ring) s_head = head + m;  // ring as per-batch scratch
        cnt_add(cnt, b, L6 + 4, m);
      }
    }
  }
  __syncthreads();
  if (tid == 0) {
    *lv.n_c_total = s_base;
    if (has_ring) {
      c.state[0] = s_head;
      c.state[1] = s_size;
      if (use_cache && c.state[3] * 10 > (long long)(c.imask + 1) * 9) atomicOr(err, kErrIndexFull);
    }
  }
}

// ---------------------------------------------- cached levels, in parallel
// The same CacheLookup/CacheStore semantics as k_probe, in three launches:
//  (1) k_probe_pre: read-only lookup of every key of the superbatch in the
//      global index (state at superbatch start) -- fully parallel;
//  (2) k_probe_seq: one thread-block cluster walks the batches in order and
//      decides hit / miss per batch against (a) keys first missed earlier in
//      this superbatch, kept in a DSMEM hash, else (b) the pre-looked-up
//      position; misses get FIFO positions head0 + q (q = rank in the
//      superbatch's compute list, since positions are handed out in order);
//  (3) k_probe_ins: parallel insert of the superbatch's misses into the
//      global index (key -> head0 + q), skipping keys re-missed later.
// The newest copy of a key is always first on its probe chain (an insert
// takes the first dead or empty slot), so lookups stop at the first match.
__device__ __forceinline__ int sbh_pre(const LevelDev& lv, int S, int* s_pre) {
  if (threadIdx.x == 0) {
    int a = 0;
    for (int b = 0; b < S; ++b) {
      s_pre[b] = a;
      a += lv.n_u[b];
    }
    s_pre[S] = a;
  }
  __syncthreads();
  return s_pre[S];
}
__device__ __forceinline__ int sbh_batch(const int* s_pre, int S, int j) {  // last b with pre[b] <= j
  int lo = 0, hi = S - 1;
  while (lo < hi) {
    const int mid = (lo + hi + 1) >> 1;
    if (s_pre[mid] <= j) lo = mid; else hi = mid - 1;
  }
  return lo;
}
__device__ __forceinline__ unsigned long long sbh_mask(const CacheDev& c, int NT) {
  unsigned long long T = 1024;
  while (T < 4ull * (unsigned long long)NT && T <= c.sb_mask) T <<= 1;  // both passes' keys: load <= 1/2
  return (T > c.sb_mask + 1 ? c.sb_mask + 1 : T) - 1;
}

__global__ void k_probe_pre(LevelDev lv, int S, CacheDev c) { pdl_enter();
  // an index rebuild (launch_index_maint, just before) left its filled-slot count in state[7]
  if (blockIdx.x == 0 && threadIdx.x == 0 &&
      c.state[3] * kIndexRebuildDen > (long long)(c.imask + 1) * kIndexRebuildNum)
    c.state[3] = c.state[7];
  if (blockIdx.x == 0 && threadIdx.x == 0 && c.occ_report) {  // one 64-bit store: consistent pair
    const unsigned long long occ = (unsigned long long)c.state[3] & ((1ull << 40) - 1);
    *(volatile unsigned long long*)c.occ_report = ((unsigned long long)(c.report_sb + 1) << 40) | occ;
    __threadfence_system();
  }
  if (c.sb_key) {  // clear the superbatch-scoped hash of the grid-wide pass (k_sbh_*)
    __shared__ int s_pre[kMaxS + 1];
    const unsigned long long T = sbh_mask(c, sbh_pre(lv, S, s_pre)) + 1;
    for (unsigned long long h = blockIdx.x * (unsigned long long)blockDim.x + threadIdx.x; h < T;
         h += (unsigned long long)gridDim.x * blockDim.x) {
      c.sb_key[h] = kEmptyKey;
      c.sb_val[h] = 0xFFFFFFFFu;
    }
  }
  const int tot = S * lv.cap;
  for (int idx = blockIdx.x * blockDim.x + threadIdx.x; idx < tot; idx += gridDim.x * blockDim.x) {
    const int b = idx / lv.cap, i = idx - b * lv.cap;
    if (i >= lv.n_u[b]) continue;
    const unsigned long long key = tkey(lv.u_node[idx], lv.u_ts[idx]);
    unsigned long long h = mix64(key) & c.imask;
    long long p = -1;
    for (unsigned long long pr = 0; pr <= c.imask; ++pr) {
      const unsigned long long k0 = __ldcg(c.ikey + h);
      if (k0 == kEmptyKey) break;
      if (k0 == key) {
        p = __ldcg(c.ipos + h);
        break;
      }
      h = (h + 1) & c.imask;
    }
    lv.p0[idx] = p;
  }
}

constexpr int kSeqCL = kSeqCLMax;
constexpr int kSeqThreads = 1024;
// k_probe_seq runs after an abandoned grid-wide attempt whose keys still occupy the superbatch
// table: its own entries carry bit 63 (node ids < 2^31 leave it clear in Hash(n, t))
constexpr unsigned long long kSeqTag = 1ull << 63;
constexpr int kSeqSlots = kSeqSlotsPerCTA;

__global__ void __launch_bounds__(kSeqThreads, 1)
k_probe_seq(LevelDev lv, int S, CacheDev c, long long* cnt, int layer, int* err) { pdl_enter();
  // key -> q of its latest miss in this superbatch: the superbatch hash in global memory
  // (L2-resident, cleared by k_probe_pre), so any S fits (r1 kept it in DSMEM, capping S)
  unsigned long long* skey = c.sb_key;
  unsigned* sq = c.sb_val;
  __shared__ int s_pre[kMaxS + 1];
  __shared__ int s_warp[32];
  __shared__ int s_total;
  __shared__ long long s_head, s_size;
  __shared__ int s_base;
  cg::cluster_group cluster = cg::this_cluster();
  const unsigned CL = cluster.num_blocks();
  const unsigned rank = cluster.block_rank();
  const int tid = threadIdx.x;
  const int NT = sbh_pre(lv, S, s_pre);
  if (c.state[5] == 1) return;  // the eviction-free parallel pass handled this superbatch
  if (rank == 0 && tid == 0) {
    s_head = __ldcg(c.state + 0);
    s_size = __ldcg(c.state + 1);
    s_base = 0;
    c.state[4] = c.state[0];  // head0 for the insert pass
  }
  const long long limit = __ldcg(c.state + 2);
  const long long head0 = __ldcg(c.state + 0);
  const unsigned long long tmask = sbh_mask(c, NT);
  cluster.sync();
  for (int b = 0; b < S; ++b) {
    const long long head = *cluster.map_shared_rank(&s_head, 0);
    const long long size = *cluster.map_shared_rank(&s_size, 0);
    const int cbase = *cluster.map_shared_rank(&s_base, 0);
    const long long live_lo = head - size;
    const int n = lv.n_u[b];
    const size_t seg = (size_t)b * lv.cap;
    const int chunk = (n + (int)CL - 1) / (int)CL;
    const int cbeg = min(n, (int)rank * chunk), cend = min(n, cbeg + chunk);
    const int ipt = (chunk + (int)blockDim.x - 1) / (int)blockDim.x;
    const int tbeg = cbeg + tid * ipt;
    int m_local = 0;
    unsigned missmask = 0;
    unsigned sbslot[kProbeIPT];
#pragma unroll
    for (int j = 0; j < kProbeIPT; ++j) {
      sbslot[j] = 0xFFFFFFFFu;
      const int i = tbeg + j;
      if (j < ipt && i < cend) {
        const unsigned long long key = tkey(lv.u_node[seg + i], lv.u_ts[seg + i]) | kSeqTag;
        long long p = -1;
        unsigned long long h = mix64(key) & tmask;
        for (unsigned long long pr = 0; pr <= tmask; ++pr) {
          const unsigned long long k0 = __ldcg(skey + h);
          if (k0 == kEmptyKey) break;
          if (k0 == key) {
            sbslot[j] = (unsigned)h;
            p = head0 + __ldcg(sq + h);
            break;
          }
          h = (h + 1) & tmask;
        }
        if (sbslot[j] == 0xFFFFFFFFu) p = __ldcg(lv.p0 + seg + i);
        if (p >= 0 && p >= live_lo) {
          lv.slot[seg + i] = p % c.rcap;  // hit (Alg. 1 l.8)
        } else {
          missmask |= 1u << j;
          ++m_local;
        }
      }
    }
    int tot_cta;
    const int excl = block_excl_scan(m_local, s_warp, tot_cta);
    if (tid == 0) s_total = tot_cta;
    cluster.sync();
    int before = 0, m = 0;
    for (unsigned r = 0; r < CL; ++r) {
      const int v = *cluster.map_shared_rank(&s_total, r);
      if (r < rank) before += v;
      m += v;
    }
    int rr = before + excl;
#pragma unroll
    for (int j = 0; j < kProbeIPT; ++j) {
      if (missmask & (1u << j)) {
        const int i = tbeg + j;
        const int q = cbase + rr;
        const int32_t node = lv.u_node[seg + i];
        const uint32_t t = lv.u_ts[seg + i];
        lv.c_b[q] = b;
        lv.c_u[q] = i;
        lv.c_node[q] = node;
        lv.c_ts[q] = t;
        lv.sup[q] = 0;
        lv.slot[seg + i] = (head + rr) % c.rcap;  // == (head0 + q) % rcap
        const unsigned long long key = tkey(node, t) | kSeqTag;
        if (sbslot[j] != 0xFFFFFFFFu) {  // evicted and missed again inside this SB
          const unsigned h = sbslot[j];
          unsigned* qp = sq + h;
          lv.sup[__ldcg(qp)] = 1;
          *qp = (unsigned)q;
        } else {
          unsigned long long h = mix64(key) & tmask;
          for (unsigned long long pr = 0; pr <= tmask; ++pr) {
            unsigned long long* kp = skey + h;
            const unsigned long long old = atomicCAS(kp, kEmptyKey, key);
            if (old == kEmptyKey || old == key) {
              sq[h] = (unsigned)q;
              break;
            }
            h = (h + 1) & tmask;
          }
        }
        ++rr;
      }
    }
    if (rank == 0 && tid == 0) {
      const long long nsz = size + m < limit ? size + m : limit;
      const long long ev_total = size + m - nsz;
      const long long evicted = ev_total < size ? ev_total : size;
      s_head = head + m;
      s_size = nsz;
      s_base = cbase + m;
      lv.c_base[b] = cbase;
      lv.n_c[b] = m;
      const int L6 = layer * TG_CNT_PER_LAYER;
      cnt_add(cnt, b, L6 + 2, n);      // lookups
      cnt_add(cnt, b, L6 + 3, n - m);  // hits
      cnt_add(cnt, b, L6 + 4, m);      // misses = embeddings computed
      cnt_add(cnt, b, L6 + 5, evicted);
    }
    cluster.sync();
  }
  if (rank == 0 && tid == 0) {
    *lv.n_c_total = s_base;
    c.state[0] = s_head;
    c.state[1] = s_size;
  }
  cluster.sync();
}

// Eviction-free superbatch (size0 + sum_b |U_b| <= limit): nothing live at
// the start or inserted during the superbatch can leave the FIFO window, so
// the sequential outcome is closed-form: the occurrence of a key in batch b
// hits iff an earlier batch of the superbatch holds the same key, or the key
// is live in the index at superbatch start. Over the concatenated unique lists
// (j = batch-major order, the order of Alg. 1's lookups), grid-wide on every SM,
// with a superbatch-scoped hash table in global memory (cleared by k_probe_pre):
//   k_sbh_insert  every key: claim a table slot (CAS on the key), atomicMin(j);
//   k_sbh_count   misses = first occurrences not live at superbatch start, per
//                 contiguous block of j;
//   k_sbh_assign  ordered rank q of every miss (block offset + block scan): its
//                 FIFO position is head0 + q; first occurrences publish their slot;
//   k_sbh_finish  later occurrences take the slot of their first; per-batch
//                 compute-list bounds, counters and the FIFO state.
// If eviction is possible the four kernels return at once and the ordered pass
// (k_probe_seq) handles the superbatch.
__global__ void k_sbh_insert(LevelDev lv, int S, CacheDev c, int* err) { pdl_enter();
  __shared__ int s_pre[kMaxS + 1];
  const int NT = sbh_pre(lv, S, s_pre);
  if (blockIdx.x == 0 && threadIdx.x == 0) {
    c.state[5] = 1;          // grid-wide pass attempted (k_sbh_finish may hand over to k_probe_seq)
    c.state[6] = LLONG_MAX;  // min index position of the superbatch's first-occurrence hits
  }
  const unsigned long long tmask = sbh_mask(c, NT);
  for (int j = blockIdx.x * blockDim.x + threadIdx.x; j < NT; j += gridDim.x * blockDim.x) {
    const int b = sbh_batch(s_pre, S, j);
    const size_t idx = (size_t)b * lv.cap + (j - s_pre[b]);
    const unsigned long long key = tkey(lv.u_node[idx], lv.u_ts[idx]);
    unsigned long long h = mix64(key) & tmask;
    int hs = -1;
    for (unsigned long long pr = 0; pr <= tmask; ++pr) {
      const unsigned long long old = atomicCAS(c.sb_key + h, kEmptyKey, key);
      if (old == kEmptyKey || old == key) {
        atomicMin(c.sb_val + h, (unsigned)j);
        hs = (int)h;
        break;
      }
      h = (h + 1) & tmask;
    }
    if (hs < 0) atomicOr(err, kErrDedupFull);
    c.sb_h[idx] = hs;
  }
}

// miss test of entry j (first occurrence, not live at superbatch start)
__device__ __forceinline__ bool sbh_first(const LevelDev& lv, const CacheDev& c, size_t idx, int j) {
  const int h = c.sb_h[idx];
  return h >= 0 && __ldcg(c.sb_val + h) == (unsigned)j;
}

__global__ void __launch_bounds__(kSbhThreads) k_sbh_count(LevelDev lv, int S, CacheDev c) { pdl_enter();
  __shared__ int s_pre[kMaxS + 1];
  __shared__ int s_warp[32];
  const int NT = sbh_pre(lv, S, s_pre);
  if (__ldcg(c.state + 5) != 1) return;
  const long long live_lo = __ldcg(c.state + 0) - __ldcg(c.state + 1);
  const int j0 = blockIdx.x * kSbhChunk + threadIdx.x * kSbhItems;
  int m = 0;
#pragma unroll
  for (int e = 0; e < kSbhItems; ++e) {
    const int j = j0 + e;
    if (j < NT) {
      const int b = sbh_batch(s_pre, S, j);
      const size_t idx = (size_t)b * lv.cap + (j - s_pre[b]);
      if (sbh_first(lv, c, idx, j)) {
        const long long p = __ldcg(lv.p0 + idx);
        m += !(p >= 0 && p >= live_lo);
      }
    }
  }
  int tot;
  block_excl_scan(m, s_warp, tot);
  if (threadIdx.x == 0) c.sb_blk[blockIdx.x] = tot;
}

__global__ void __launch_bounds__(kSbhThreads) k_sbh_assign(LevelDev lv, int S, CacheDev c) { pdl_enter();
  __shared__ int s_pre[kMaxS + 1];
  __shared__ int s_warp[32];
  __shared__ int s_off;
  const int NT = sbh_pre(lv, S, s_pre);
  if (__ldcg(c.state + 5) != 1) return;
  const long long head0 = __ldcg(c.state + 0);
  const long long live_lo = head0 - __ldcg(c.state + 1);
  if (threadIdx.x == 0) {
    int o = 0;
    for (int q = 0; q < (int)blockIdx.x; ++q) o += __ldcg(c.sb_blk + q);
    s_off = o;
  }
  const int j0 = blockIdx.x * kSbhChunk + threadIdx.x * kSbhItems;
  unsigned first = 0, miss = 0;
  int m = 0;
#pragma unroll
  for (int e = 0; e < kSbhItems; ++e) {
    const int j = j0 + e;
    if (j < NT) {
      const int b = sbh_batch(s_pre, S, j);
      const size_t idx = (size_t)b * lv.cap + (j - s_pre[b]);
      if (sbh_first(lv, c, idx, j)) {
        first |= 1u << e;
        const long long p = __ldcg(lv.p0 + idx);
        if (!(p >= 0 && p >= live_lo)) {
          miss |= 1u << e;
          ++m;
        }
      }
    }
  }
  int tot;
  const int excl = block_excl_scan(m, s_warp, tot);  // (syncs: s_off visible)
  int q = s_off + excl;
  long long pmin = LLONG_MAX;  // min index position of this thread's first-occurrence hits
#pragma unroll
  for (int e = 0; e < kSbhItems; ++e) {
    if (!(first & (1u << e))) continue;
    const int j = j0 + e;
    const int b = sbh_batch(s_pre, S, j);
    const int u = j - s_pre[b];
    const size_t idx = (size_t)b * lv.cap + u;
    long long sl;
    if (miss & (1u << e)) {
      lv.c_b[q] = b;
      lv.c_u[q] = u;
      lv.c_node[q] = lv.u_node[idx];
      lv.c_ts[q] = lv.u_ts[idx];
      lv.sup[q] = 0;
      sl = (head0 + q) % c.rcap;
      ++q;
    } else {
      const long long p = __ldcg(lv.p0 + idx);
      pmin = p < pmin ? p : pmin;
      sl = p % c.rcap;
    }
    lv.slot[idx] = sl;
    c.sb_slot[c.sb_h[idx]] = sl;
  }
  // one atomic per warp (a single hot address otherwise serialises the whole grid)
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    const long long other = __shfl_xor_sync(0xffffffffu, pmin, o);
    pmin = other < pmin ? other : pmin;
  }
  if ((threadIdx.x & 31) == 0 && pmin != LLONG_MAX) atomicMin(reinterpret_cast<long long*>(c.state + 6), pmin);
}

__global__ void k_sbh_finish(LevelDev lv, int S, CacheDev c, long long* cnt, int layer, int nblk) { pdl_enter();
  __shared__ int s_pre[kMaxS + 1];
  __shared__ int s_M;
  const int NT = sbh_pre(lv, S, s_pre);
  if (__ldcg(c.state + 5) != 1) return;
  // later occurrences: the slot of the first one (Alg. 1 l.8 hit inside the superbatch)
  for (int j = blockIdx.x * blockDim.x + threadIdx.x; j < NT; j += gridDim.x * blockDim.x) {
    const int b = sbh_batch(s_pre, S, j);
    const size_t idx = (size_t)b * lv.cap + (j - s_pre[b]);
    if (!sbh_first(lv, c, idx, j)) lv.slot[idx] = __ldcg(c.sb_slot + c.sb_h[idx]);
  }
  if (blockIdx.x != 0) return;
  __shared__ int s_ok;
  if (threadIdx.x == 0) {
    int M = 0;
    for (int q = 0; q < nblk; ++q) M += __ldcg(c.sb_blk + q);
    s_M = M;
    // The closed form is the sequential outcome iff nothing it counts as a hit leaves the FIFO
    // window before its batch: every first-occurrence hit's position must still be live after
    // the superbatch's last store, and no in-superbatch miss may be evicted (M <= limit).
    // Otherwise the ordered pass (k_probe_seq) redoes the superbatch batch by batch.
    const long long head0 = c.state[0], size0 = c.state[1], limit = c.state[2];
    const long long live_lo_end = head0 + M - (size0 + M < limit ? size0 + M : limit);
    s_ok = (M <= limit && __ldcg(c.state + 6) >= live_lo_end) ? 1 : 0;
    if (!s_ok) c.state[5] = 0;
  }
  __syncthreads();
  if (!s_ok) return;
  const int M = s_M;
  if (threadIdx.x < S) {
    // misses of batch b = misses with j in [pre[b], pre[b+1]): bounds in the compute list
    const int b = threadIdx.x;
    int lo = 0, hi = M;  // first q with c_b[q] >= b
    while (lo < hi) {
      const int mid = (lo + hi) >> 1;
      if (__ldcg(lv.c_b + mid) < b) lo = mid + 1; else hi = mid;
    }
    int lo2 = lo, hi2 = M;  // first q with c_b[q] > b
    while (lo2 < hi2) {
      const int mid = (lo2 + hi2) >> 1;
      if (__ldcg(lv.c_b + mid) <= b) lo2 = mid + 1; else hi2 = mid;
    }
    const int n = s_pre[b + 1] - s_pre[b], m = lo2 - lo;
    lv.c_base[b] = lo;
    lv.n_c[b] = m;
    const int L6 = layer * TG_CNT_PER_LAYER;
    cnt_add(cnt, b, L6 + 2, n);      // lookups
    cnt_add(cnt, b, L6 + 3, n - m);  // hits
    cnt_add(cnt, b, L6 + 4, m);      // misses
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    const long long head0 = c.state[0], size0 = c.state[1], limit = c.state[2];
    long long size = size0;
    for (int b = 0; b < S; ++b) {  // FIFO sizes and evictions batch by batch (R11, R19)
      const long long m = lv.n_c[b];
      const long long nsz = size + m < limit ? size + m : limit;
      const long long ev_total = size + m - nsz;
      cnt_add(cnt, b, layer * TG_CNT_PER_LAYER + 5, ev_total < size ? ev_total : size);
      size = nsz;
    }
    *lv.n_c_total = M;
    c.state[4] = head0;
    c.state[0] = head0 + M;
    c.state[1] = size;
  }
}

// No lookup (top layer, R9; or cache disabled): C = the unique lists of the S
// batches concatenated in batch order, q = c_base[b] + u. With a ring (cache
// disabled at a cached level) the rows still go to FIFO positions head + q,
// used as per-superbatch scratch.
__global__ void k_compact_all(LevelDev lv, int S, CacheDev c, int has_ring, long long* cnt, int layer) { pdl_enter();
  __shared__ int s_pre[kMaxS + 1];
  if (threadIdx.x == 0) {
    int a = 0;
    for (int b = 0; b < S; ++b) {
      s_pre[b] = a;
      a += lv.n_u[b];
    }
    s_pre[S] = a;
  }
  __syncthreads();
  const long long head = has_ring ? c.state[0] : 0;
  const int tot = S * lv.cap;
  for (int idx = blockIdx.x * blockDim.x + threadIdx.x; idx < tot; idx += gridDim.x * blockDim.x) {
    const int b = idx / lv.cap, u = idx - b * lv.cap;
    if (u >= s_pre[b + 1] - s_pre[b]) continue;
    const int q = s_pre[b] + u;
    lv.c_b[q] = b;
    lv.c_u[q] = u;
    lv.c_node[q] = lv.u_node[idx];
    lv.c_ts[q] = lv.u_ts[idx];
    if (has_ring) lv.slot[idx] = (head + q) % c.rcap;
  }
  if (blockIdx.x == 0) {
    for (int b = threadIdx.x; b < S; b += blockDim.x) {
      const int m = s_pre[b + 1] - s_pre[b];
      lv.c_base[b] = s_pre[b];
      lv.n_c[b] = m;
      cnt_add(cnt, b, layer * TG_CNT_PER_LAYER + 4, m);  // misses = embeddings computed
    }
    __syncthreads();
    if (threadIdx.x == 0) {
      *lv.n_c_total = s_pre[S];
      // every block has read head before the grid ends; the next launch sees the update
    }
  }
}

// head update of the scratch ring after k_compact_all (separate launch: no
// intra-grid ordering needed)
__global__ void k_ring_advance(LevelDev lv, CacheDev c) { pdl_enter(); c.state[0] += *lv.n_c_total; }

__global__ void k_probe_ins(LevelDev lv, CacheDev c, int* err) { pdl_enter();
  const int n = *lv.n_c_total;
  const long long head0 = __ldcg(c.state + 4);
  const long long live_lo = __ldcg(c.state + 0) - __ldcg(c.state + 1);
  for (int q = blockIdx.x * blockDim.x + threadIdx.x; q < n; q += gridDim.x * blockDim.x) {
    const unsigned long long key = tkey(lv.c_node[q], lv.c_ts[q]);
    const long long pos = head0 + q;
    c.rkey[pos % c.rcap] = key;  // for index rebuilds
    // Skip superseded misses and misses already evicted by the end of this superbatch
    // (pos < live_lo: more misses than the limit, R11). Inserting a dead-on-arrival key
    // would let its slot be locked and rewritten twice in this launch (dead -> dead ->
    // live), an ABA under which a thread still holding the slot's first key could CAS
    // over the live key written last. Every write below makes its slot live, and live
    // slots are never reusable within the launch.
    if (lv.sup[q] || pos < live_lo) continue;
    unsigned long long h = mix64(key) & c.imask;
    bool done = false;
    for (unsigned long long pr = 0; pr <= 4 * c.imask && !done; ++pr) {
      const unsigned long long k0 = ld_volatile_u64(c.ikey + h);
      if (k0 != kLockedKey) {
        __threadfence();
        const bool reusable = (k0 == kEmptyKey) || (k0 == key) || (*(volatile long long*)(c.ipos + h) < live_lo);
        if (reusable) {
          if (atomicCAS(c.ikey + h, k0, kLockedKey) == k0) {
            // Re-check under the lock: the CAS only proves ikey still equals k0, not that
            // the slot is still dead. A concurrent re-insert of the dead key k0 itself (k0
            // evicted earlier, missed again in this superbatch) can lock, write a live
            // position and unlock with the same key value between our ipos read and our
            // CAS -- an ABA that used to overwrite k0's live entry (that key then missed
            // once while still in the FIFO window). ipos only changes under the lock.
            __threadfence();
            if (k0 != kEmptyKey && k0 != key && *(volatile long long*)(c.ipos + h) >= live_lo) {
              atomicExch(c.ikey + h, k0);  // live after all: release unchanged, probe on
              h = (h + 1) & c.imask;
              continue;
            }
            *(volatile long long*)(c.ipos + h) = pos;
            __threadfence();
            atomicExch(c.ikey + h, key);
            if (k0 == kEmptyKey) atomicAdd((unsigned long long*)(c.state + 3), 1ull);
            done = true;
          }
          continue;
        }
      }
      h = (h + 1) & c.imask;
    }
    if (!done) atomicOr(err, kErrIndexFull);
  }
}

// Index rebuild, phase 1: clear (every CTA takes the same decision from state[3],
// which nothing modifies until k_probe_pre).
__global__ void k_index_clear(CacheDev c) { pdl_enter();
  if (!(c.state[3] * kIndexRebuildDen > (long long)(c.imask + 1) * kIndexRebuildNum)) return;
  const unsigned long long n = c.imask + 1;
  for (unsigned long long i = blockIdx.x * (unsigned long long)blockDim.x + threadIdx.x; i < n;
       i += (unsigned long long)gridDim.x * blockDim.x) {
    c.ikey[i] = kEmptyKey;
    c.ipos[i] = -1;
  }
  if (blockIdx.x == 0 && threadIdx.x == 0) c.state[7] = 0;
}
// phase 2: re-insert the live window [head - size, head); a key present several
// times keeps its newest position (atomicMax), as the sequential inserts did.
__global__ void k_index_reinsert(CacheDev c, int* err) { pdl_enter();
  if (!(c.state[3] * kIndexRebuildDen > (long long)(c.imask + 1) * kIndexRebuildNum)) return;
  const long long head = c.state[0], lo = head - c.state[1];
  for (long long p = lo + blockIdx.x * (long long)blockDim.x + threadIdx.x; p < head;
       p += (long long)gridDim.x * blockDim.x) {
    const unsigned long long key = c.rkey[p % c.rcap];
    unsigned long long h = mix64(key) & c.imask;
    bool done = false;
    for (unsigned long long pr = 0; pr <= c.imask && !done; ++pr) {
      const unsigned long long k0 = atomicCAS(c.ikey + h, kEmptyKey, key);
      if (k0 == kEmptyKey || k0 == key) {
        atomicMax(c.ipos + h, p);
        if (k0 == kEmptyKey) atomicAdd((unsigned long long*)(c.state + 7), 1ull);
        done = true;
      }
      h = (h + 1) & c.imask;
    }
    if (!done) atomicOr(err, kErrIndexFull);
  }
}

// debug (TG_DBG_INDEX_CHECK=1): every key of the live window must be found at its newest
// position; mismatches are counted into err[1]
__global__ void k_index_check(CacheDev c, int* err) {
  const long long head = c.state[0], lo = head - c.state[1];
  for (long long p = lo + blockIdx.x * (long long)blockDim.x + threadIdx.x; p < head;
       p += (long long)gridDim.x * blockDim.x) {
    const unsigned long long key = c.rkey[p % c.rcap];
    // newest position of this key within the window: scan forward is too slow; check that
    // the index position is >= p (the newest copy is never older than any live copy)
    unsigned long long h = mix64(key) & c.imask;
    long long found = -2;
    for (unsigned long long pr = 0; pr <= c.imask; ++pr) {
      const unsigned long long k0 = __ldcg(c.ikey + h);
      if (k0 == kEmptyKey) { found = -1; break; }
      if (k0 == key) { found = __ldcg(c.ipos + h); break; }
      h = (h + 1) & c.imask;
    }
    if (found < p) atomicAdd(err + 1, 1);
  }
}
void launch_index_check(const CacheDev& c, int* err, cudaStream_t st) {
  k_index_check<<<148, 256, 0, st>>>(c, err);
}

int launch_index_maint(const CacheDev& c, cudaStream_t st, int* err) {
  launch_k(k_index_clear, dim3(148 * 4), dim3(256), 0, st, c);
  launch_k(k_index_reinsert, dim3(148 * 4), dim3(256), 0, st, c, err);
  return 2;
}

int launch_probe(LevelDev lv, int S, const CacheDev* cache, long long* cnt, int layer, int* err,
                 cudaStream_t st) {
  CacheDev c{};
  int has_ring = 0, use_cache = 0;
  if (cache) {
    c = *cache;
    has_ring = 1;
    use_cache = c.ikey != nullptr;
  }
  if (!use_cache) {  // top layer (no lookup, R9) or cache disabled: every unique entry is computed
    int blocks = (S * lv.cap + 255) / 256;
    if (blocks > 148 * 4) blocks = 148 * 4;
    if (blocks < 1) blocks = 1;
    launch_k(k_compact_all, dim3(blocks), dim3(256), 0, st, lv, S, c, has_ring, cnt, layer);
    if (has_ring) {
      launch_k(k_ring_advance, dim3(1), dim3(1), 0, st, lv, c);
      return 2;
    }
    return 1;
  }
  int blocks = (S * lv.cap + 255) / 256;
  if (blocks > 148 * 8) blocks = 148 * 8;
  launch_k(k_probe_pre, dim3(blocks), dim3(256), 0, st, lv, S, c);
  static bool attr = false;
  if (!attr) {
    cudaFuncSetAttribute(k_probe_seq, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
    attr = true;
  }
  // the ordered pass walks one batch at a time: enough CTAs for <= 4 keys per thread
  int cl = 1;
  while (cl < kSeqCL && (long long)cl * kSeqThreads * 4 < (long long)lv.cap) cl <<= 1;
  // eviction-free superbatches: grid-wide pass (k_sbh_*); otherwise the ordered pass
  const int nj = S * lv.cap;
  int gb = (nj + 255) / 256;
  if (gb > 148 * 8) gb = 148 * 8;
  const int nblk = (nj + kSbhChunk - 1) / kSbhChunk;
  launch_k(k_sbh_insert, dim3(gb), dim3(256), 0, st, lv, S, c, err);
  launch_k(k_sbh_count, dim3(nblk), dim3(kSbhThreads), 0, st, lv, S, c);
  launch_k(k_sbh_assign, dim3(nblk), dim3(kSbhThreads), 0, st, lv, S, c);
  launch_k(k_sbh_finish, dim3(gb), dim3(256), 0, st, lv, S, c, cnt, layer, nblk);
  launch_k_cluster(k_probe_seq, dim3(cl), dim3(kSeqThreads), 0, st, cl, lv, S, c, cnt, layer, err);
  int ib = (S * lv.cap + 255) / 256;
  if (ib > 148 * 4) ib = 148 * 4;
  launch_k(k_probe_ins, dim3(ib), dim3(256), 0, st, lv, c, err);
  return 7;
}

// ------------------------------------------------------------------ NghLookup
// Warp per target q: 32-ary search for the first adjacency entry with
// t_j >= t (strict t_j < t), then lanes copy the last min(k, p-lo)
// entries right-aligned (R6), padding (0, 0, 0) on the left (R7). Writes the
// compute-centric neighbour slots and the next level's input list
// I_{l-1} = [C_l ; N(C_l)] of each batch (Alg. 1 l.12). Also counts, per
// batch, how many Phi(dt) the precomputed window serves (Sec. 4.3).
__global__ void k_sample(GraphDev g, LevelDev lv, int S, int k, LevelDev nx, int has_next, int W, int use_table,
                         long long* cnt, int layer, int* err) { pdl_enter();
  const int lane = threadIdx.x & 31;
  const int warp = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int nwarps = (gridDim.x * blockDim.x) >> 5;
  if (blockIdx.x == 0 && threadIdx.x < S) {
    const int b = threadIdx.x;
    const int nb = lv.n_c[b];
    if (has_next) nx.n_in[b] = nb * (k + 1);
    if (layer == 1) cnt_add(cnt, b, 0, (long long)nb * (k + 1));  // h^(0) lookups (l0 n)
  }
  const int nC = *lv.n_c_total;
  for (int q = warp; q < nC; q += nwarps) {
    const int b = lv.c_b[q];
    const int p = q - lv.c_base[b];
    const int nb = lv.n_c[b];
    int i = lv.c_node[q];
    const uint32_t t = lv.c_ts[q];
    if (i < 0 || i > g.V) {
      if (lane == 0) atomicOr(err, kErrNodeRange);
      i = 0;
    }
    int a = g.rowptr[i], bnd = g.rowptr[i + 1];
    const int lo = a;
    // invariant: the first entry with t_j >= t lies in [a, bnd] (bnd = "none")
    while (bnd - a > 31) {
      const int step = (bnd - a + 31) >> 5;
      const int x = a + lane * step;
      const bool ge = (x < bnd) ? (g.adj_t[x] >= t) : true;
      const unsigned msk = __ballot_sync(0xffffffffu, ge);
      if (msk == 0) {
        a = a + 31 * step + 1;
        continue;
      }
      const int f = __ffs(msk) - 1;
      const int nbd = a + f * step;
      a = (f == 0) ? a : a + (f - 1) * step + 1;
      bnd = nbd < bnd ? nbd : bnd;
    }
    {
      const int x = a + lane;  // bnd - a <= 31: lane (bnd - a) votes true
      const bool ge = (x < bnd) ? (g.adj_t[x] >= t) : true;
      const unsigned msk = __ballot_sync(0xffffffffu, ge);
      a = a + (__ffs(msk) - 1);
    }
    const int c = min(k, a - lo);
    int nbr = 0, e = 0;
    uint32_t tj = 0;
    if (lane < k && lane >= k - c) {
      const int x = a - k + lane;
      nbr = g.adj_nbr[x];
      e = g.adj_eid[x];
      tj = g.adj_t[x];
    }
    if (lane < k) {
      const size_t o = (size_t)q * k + lane;
      lv.nb_node[o] = nbr;
      lv.nb_ts[o] = tj;
      lv.nb_eid[o] = e;
      if (has_next) {
        const size_t seg = (size_t)b * nx.cap;
        nx.in_node[seg + nb + (size_t)p * k + lane] = nbr;
        nx.in_ts[seg + nb + (size_t)p * k + lane] = tj;
      }
    }
    if (lane == 0 && has_next) {
      const size_t seg = (size_t)b * nx.cap;
      nx.in_node[seg + p] = lv.c_node[q];
      nx.in_ts[seg + p] = t;
    }
    // Phi(t - t_j) source per slot: table if dt < W (padding: t_j = 0, dt = t)
    const long long dt = (long long)t - (long long)tj;
    const unsigned tab = __ballot_sync(0xffffffffu, lane < k && use_table && dt < W);
    if (lane == 0) {
      const int nt = __popc(tab);
      cnt_add(cnt, b, TG_CNT_TTABLE, nt);
      cnt_add(cnt, b, TG_CNT_TDIRECT, k - nt);
    }
  }
}

void launch_sample(const GraphDev& g, LevelDev lv, int S, int k, const LevelDev* next, int W, int use_table,
                   long long* cnt, int layer, int* err, cudaStream_t st) {
  int blocks = (lv.c_cap * 32 + 255) / 256;
  if (blocks < 1) blocks = 1;
  if (blocks > 148 * 8) blocks = 148 * 8;
  LevelDev nx{};
  if (next) nx = *next;
  launch_k(k_sample, dim3(blocks), dim3(256), 0, st, g, lv, S, k, nx, next ? 1 : 0, W, use_table, cnt, layer, err);
}

// ---------------------------------------------------------------- row lookup
// Layer l reads h^(l-1): x_i at l = 1 (Alg. 1 l.2-3), else the ring
// slot of the target's unique entry at level l-1 (through inv, Alg. 1 l.20).
__global__ void k_resolve(ResolveArgs a, int* err) { pdl_enter();
  const int l = blockIdx.y + 1;
  const LevelDev& lv = a.lv[l];
  const LevelDev& pv = a.lv[l - 1];
  const int k = a.k;
  const int n = *lv.n_c_total;
  const long long tot = (long long)n * (k + 1);
  for (long long idx = blockIdx.x * (long long)blockDim.x + threadIdx.x; idx < tot;
       idx += (long long)gridDim.x * blockDim.x) {
    const int q = (int)(idx / (k + 1));
    const int m = (int)(idx - (long long)q * (k + 1)) - 1;
    const int b = lv.c_b[q];
    const int p = q - lv.c_base[b];
    if (m < 0) {
      const float* hs;
      if (l == 1) {
        int node = lv.c_node[q];
        if (node < 0) {
          atomicOr(err, kErrNodeRange);
          node = 0;
        }
        hs = a.X + (size_t)node * a.ldn;
      } else {
        const size_t seg = (size_t)b * pv.cap;
        hs = a.ring[l - 1] + (size_t)pv.slot[seg + pv.inv[seg + p]] * a.ldn;
      }
      lv.hs_row[q] = hs;
      lv.dst_row[q] = (l < a.L) ? a.ring[l] + (size_t)lv.slot[(size_t)b * lv.cap + lv.c_u[q]] * a.ldn
                                : a.HL + (size_t)q * a.ldn;
    } else {
      const size_t o = (size_t)q * k + m;
      long long row;
      const float* base;
      if (l == 1) {
        int node = lv.nb_node[o];
        if (node < 0) {
          atomicOr(err, kErrNodeRange);
          node = 0;
        }
        row = node;
        base = a.X;
      } else {
        const int nb = lv.n_c[b];
        const size_t seg = (size_t)b * pv.cap;
        row = pv.slot[seg + pv.inv[seg + nb + (size_t)p * k + m]];
        base = a.ring[l - 1];
      }
      lv.nb_row[o] = base + (size_t)row * a.ldn;
      lv.nb_hidx[o] = (int32_t)row;
    }
  }
}

__global__ void k_gather_hs(ResolveArgs a, int l0) { pdl_enter();
  const int l = blockIdx.y + l0;
  const LevelDev& lv = a.lv[l];
  if (!lv.hs_dense) return;
  const int n = *lv.n_c_total;
  const int lane = threadIdx.x & 31;
  const int nq = a.ldn >> 2;
  for (int q = (blockIdx.x * blockDim.x + threadIdx.x) >> 5; q < n; q += (gridDim.x * blockDim.x) >> 5) {
    const float4* src = reinterpret_cast<const float4*>(lv.hs_row[q]);
    float4* dst = reinterpret_cast<float4*>(lv.hs_dense + (size_t)q * a.ldn);
    for (int c = lane; c < nq; c += 32) dst[c] = src[c];
  }
}

void launch_gather_hs(const ResolveArgs& a, int l0, int l1, cudaStream_t st) {
  launch_k(k_gather_hs, dim3(dim3(148 * 2, l1 - l0 + 1)), dim3(256), 0, st, a, l0);
}

void launch_resolve(const ResolveArgs& a, int* err, cudaStream_t st) {
  long long mx = (long long)a.c_cap_max * (a.k + 1);
  int bx = (int)((mx + 255) / 256);
  if (bx < 1) bx = 1;
  if (bx > 592) bx = 592;
  launch_k(k_resolve, dim3(dim3(bx, a.L)), dim3(256), 0, st, a, err);
}

// ------------------------------------------------------------------- misc
__global__ void k_prep_nodes(const int32_t* __restrict__ nodes, const uint32_t* __restrict__ ts, int n,
                             LevelDev top) { pdl_enter();
  for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) {
    top.in_node[i] = nodes[i];
    top.in_ts[i] = ts[i];
  }
  if (blockIdx.x == 0 && threadIdx.x == 0) top.n_in[0] = n;
}

void launch_prep_nodes(const int32_t* nodes, const uint32_t* ts, int n, LevelDev top, cudaStream_t st) {
  int blocks = n > 0 ? (n + 255) / 256 : 1;
  if (blocks > 592) blocks = 592;
  launch_k(k_prep_nodes, dim3(blocks), dim3(256), 0, st, nodes, ts, n, top);
}

__global__ void k_finish(long long* __restrict__ cnt_sb, int S, long long* __restrict__ total,
                         long long* __restrict__ log, int64_t row0) { pdl_enter();
  for (int i = threadIdx.x; i < S * TG_NCOUNTERS; i += blockDim.x) {
    const long long v = cnt_sb[i];
    if (v) atomicAdd((unsigned long long*)(total + i % TG_NCOUNTERS), (unsigned long long)v);
    if (log) log[row0 * TG_NCOUNTERS + i] = v;
    cnt_sb[i] = 0;
  }
}

void launch_finish(long long* cnt_sb, int S, long long* total, long long* log, int64_t log_row0,
                   cudaStream_t st) {
  launch_k(k_finish, dim3(1), dim3(1024), 0, st, cnt_sb, S, total, log, log_row0);
}

}  // namespace tg
