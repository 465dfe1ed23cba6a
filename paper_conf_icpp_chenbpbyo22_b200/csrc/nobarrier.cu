// nobarrier.cu -- NEXT-4: barrier-free partitioned PageRank and BFS.
//
// The exchange-round path (relax.cu pagerank_partitioned) runs every partition to local
// quiescence, then exchanges ghost mass and starts the next round.  Here the barrier goes away, which is
// the paper's relaxed-barrier thesis applied across partitions: one persistent kernel in
// which every partition's workers push mass for a REMOTE vertex straight into the owner's residue slice
// (atomicAdd on the owner's memory -- peer memory over NVLink in a multi-GPU build, the same device in
// this loopback build) and, on a threshold crossing (Alg.4, R-PR-7), into the owner's queue.
// Termination is global quiescence: sum(done) == sum(tail) over all partitions, read as every done
// counter and then every tail counter (monotone counters; an item's pushes are reserved before its done
// increment, so equal sums imply a moment with nothing queued or in flight anywhere).
//
// BFS runs the same kernel with Alg.2's relax: atomicMin on the owner's depth slice, activation
// on improvement gated by the owner's in-queue bit (cleared by the popper before it reads the depth).
//
// Worker: a CTA claims up to 256 items of one of its partition's S sub-queue rings (one CAS on head,
// never past tail), each thread begins one item (atomicExch residue -> rank, delta = alpha*rho/deg,
// Alg.4), and the CTA expands the batch's rows load-balanced (block scan + search, so a hub is
// split over 256 threads).  Pushes are warp-aggregated per destination partition (match_any + one
// atomicAdd on that sub-queue's tail).  Slots carry a lap tag so a consumer never mistakes the previous
// lap's value for its own item.
#include "internal.h"

namespace atos {

namespace {

constexpr uint32_t kNbMaxParts = 8;
constexpr int kNbBlock = 256;
constexpr int kNbU = 4;  // edges in flight per lane
#ifndef ATOS_NB_MINB
#define ATOS_NB_MINB 4  // CTAs per SM the register budget is sized for (64 registers)
#endif

struct NbCtl {  // one per partition; each counter on its own 128-byte line
  unsigned long long head, pad0[15];
  unsigned long long tail, pad1[15];
  unsigned long long done, pad2[15];
};

struct NbPeer {  // what a partition exposes to its peers (peer-mapped in a multi-GPU build)
  const uint32_t* row_ptr;  // n_local + 1, local offsets
  const uint32_t* col;      // GLOBAL ids
  double* rank;             // n_local (caller's output slice)
  double* res;              // n_local
  unsigned long long* ring; // cap slots: 0 = free, else tag(idx) << 32 | local id
  NbCtl* ctl;
  unsigned long long mask;  // cap - 1
  uint32_t n_local, pad;
  uint32_t* depth;          // BFS: n_local (caller's output slice)
  uint32_t* inq;            // BFS: in-queue bitmap, one bit per local vertex (dedupe)
};

struct NbGlob {
  unsigned long long abort;  // 1: no-progress watchdog, 2: cfg.timeout_s deadline passed
  unsigned long long edges;  // neighbour-list entries visited
};

struct NbParams {
  const NbPeer* peers;  // device array [P]
  NbGlob* glob;
  uint32_t P, B;        // partitions, block size ceil(n / P) (atos_partition_range)
  int shift;            // log2(B) when B is a power of two, else -1
  uint32_t S;           // sub-queues per partition (each its own ring + counters; fewer CTAs per head)
  double alpha, eps;
  unsigned long long watchdog_ns;
  unsigned long long timeout_ns;  // cfg.timeout_s as a device deadline from kernel start (0: none)
  int self;                       // -1: loopback (this kernel serves every partition); else the only
                                  // partition this process serves (one partition per process, peers mapped)
};

__device__ __forceinline__ unsigned long long nb_tag(unsigned long long idx, uint32_t item) {
  // lap tag never 0 (bit 31 set), distinct for idx and idx - cap while cap < 2^31
  const unsigned long long t = (idx & 0x7FFFFFFFull) | 0x80000000ull;
  return (t << 32) | item;
}

__device__ __forceinline__ bool nb_aborted(const NbGlob* g) {
  return ld_relaxed(&g->abort) != 0ull;
}

// Warp-aggregated push of `lw` into partition `o`'s ring for the lanes with act set.
__device__ __forceinline__ void nb_push(const NbParams& prm, bool act, uint32_t o, uint32_t lw) {
  const unsigned am = __ballot_sync(0xffffffffu, act);
  if (!am || !act) return;
  const unsigned grp = __match_any_sync(am, o);
  const uint32_t lane = lane_id();
  const int leader = __ffs(grp) - 1;
  const uint32_t rank = __popc(grp & ((1u << lane) - 1u));
  const NbPeer* pe = prm.peers + o;
  const uint32_t sub = (blockIdx.x * (blockDim.x >> 5) + warp_id()) % prm.S;  // uniform per warp
  NbCtl* c = pe->ctl + sub;
  unsigned long long base = 0;
  if ((int)lane == leader) base = atomicAdd(&c->tail, (unsigned long long)__popc(grp));
  base = __shfl_sync(grp, base, leader);
  const unsigned long long idx = base + rank;
  unsigned long long* slot = pe->ring + sub * (pe->mask + 1) + (idx & pe->mask);
  // the previous lap's consumer may not have released the slot yet
  while (ld_relaxed(slot) != 0ull) {
    if (nb_aborted(prm.glob)) return;
    __nanosleep(32);
  }
  st_release(slot, nb_tag(idx, lw));
}

}  // namespace

// Rank / residue init of every partition this process serves (Alg.3, R-PR-init): rank = 1 - alpha,
// residue = 0.
__global__ void k_nb_init_vertices(NbParams prm, double one_minus_alpha) {
  const uint32_t p0 = prm.self < 0 ? 0u : (uint32_t)prm.self, p1 = prm.self < 0 ? prm.P : p0 + 1;
  for (uint32_t p = p0; p < p1; ++p) {
    const NbPeer pe = prm.peers[p];
    for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < pe.n_local;
         v += (int64_t)gridDim.x * blockDim.x) {
      pe.rank[v] = one_minus_alpha;
      pe.res[v] = 0.0;
    }
  }
}

// residue[w] += alpha*(1-alpha)/deg(v) for every edge v -> w, written into the owner's slice (warp per row).
__global__ void k_nb_init_edges(NbParams prm, uint32_t p, double c) {
  const NbPeer pe = prm.peers[p];
  const uint32_t lane = lane_id();
  const int64_t warps = (int64_t)gridDim.x * (blockDim.x >> 5);
  for (int64_t v = blockIdx.x * (int64_t)(blockDim.x >> 5) + warp_id(); v < pe.n_local; v += warps) {
    const uint32_t s = __ldg(pe.row_ptr + v), deg = __ldg(pe.row_ptr + v + 1) - s;
    if (!deg) continue;
    const double add = c / (double)deg;
    for (uint32_t e = lane; e < deg; e += 32) {
      const uint32_t w = __ldg(pe.col + s + e);
      const uint32_t o = w / prm.B;
      red_add_f64(prm.peers[o].res + (w - o * prm.B), add);
    }
  }
}

// Initial frontier of partition p: every local vertex with residue > eps (R-PR-7).
__global__ void k_nb_seed(NbParams prm, uint32_t p) {
  const uint32_t n = prm.peers[p].n_local;
  const double* res = prm.peers[p].res;
  const uint32_t stride = gridDim.x * blockDim.x;
  for (uint32_t base = blockIdx.x * blockDim.x; base < n; base += stride) {
    const uint32_t v = base + threadIdx.x;
    nb_push(prm, v < n && res[v] > prm.eps, p, v);
  }
}

// The persistent barrier-free worker kernel (one cooperative launch; CTA b serves sub-queue b % (P*S), i.e.
// partition (b % (P*S)) / S).
// A CTA claims up to kNbBlock items of its partition's ring with ONE CAS (fewer contenders on head than
// a claim per warp) and expands them as the paper's CTA worker with LBS does.
template <bool kBfs>
__global__ void __launch_bounds__(kNbBlock, ATOS_NB_MINB) k_nobarrier(NbParams prm) {
  __shared__ unsigned long long s_h;
  __shared__ uint32_t s_k;
  __shared__ int s_quit;
  __shared__ uint32_t s_off[kNbBlock], s_start[kNbBlock], s_wsum[kNbBlock / 32];
  __shared__ double s_delta[kNbBlock];
  const uint32_t q = prm.self < 0 ? blockIdx.x % (prm.P * prm.S) : (uint32_t)prm.self * prm.S + blockIdx.x % prm.S;
  const uint32_t me = q / prm.S, sub0 = q % prm.S;
  const NbPeer self = prm.peers[me];
  __shared__ uint32_t s_sq;
  const uint32_t lane = lane_id(), wid = warp_id();
  unsigned long long edges = 0, t_idle = 0, last_done = 0;
  const unsigned long long t_start = globaltimer();
  while (true) {
    if (threadIdx.x == 0) {
      // cfg.timeout_s: a device deadline, so the kernel stops on its own (the host never returns while it
      // still writes the caller's output or the rings)
      if (prm.timeout_ns && globaltimer() - t_start > prm.timeout_ns) atomicCAS(&prm.glob->abort, 0ull, 2ull);
      uint32_t k = 0, sq = sub0;
      unsigned long long h = 0;
      // own sub-queue first, then the partition's other sub-queues
      for (uint32_t i = 0; i < prm.S && k == 0; ++i) {
        sq = (sub0 + i) % prm.S;
        NbCtl* c = self.ctl + sq;
        unsigned long long hh = ld_relaxed(&c->head);
        while (true) {
          const unsigned long long t = ld_relaxed(&c->tail);
          if (hh >= t) break;
          const uint32_t want = (uint32_t)min((unsigned long long)kNbBlock, t - hh);
          const unsigned long long got = atomicCAS(&c->head, hh, hh + want);
          if (got == hh) {
            h = hh;
            k = want;
            break;
          }
          hh = got;
        }
      }
      int quit = 0;
      if (k == 0) {
        if (nb_aborted(prm.glob)) {
          quit = 1;
        } else {
          unsigned long long D = 0, T = 0;
          for (uint32_t p = 0; p < prm.P; ++p)
            for (uint32_t j = 0; j < prm.S; ++j) D += atom_read(&prm.peers[p].ctl[j].done);
          for (uint32_t p = 0; p < prm.P; ++p)
            for (uint32_t j = 0; j < prm.S; ++j) T += atom_read(&prm.peers[p].ctl[j].tail);
          if (D == T) {
            quit = 1;
          } else {
            // watchdog: no partition completed an item for watchdog_ns
            const unsigned long long now = globaltimer();
            if (t_idle == 0 || D != last_done) {
              t_idle = now;
              last_done = D;
            } else if (now - t_idle > prm.watchdog_ns) {
              atomicExch(&prm.glob->abort, 1ull);
              quit = 1;
            }
            __nanosleep(256);
          }
        }
      } else {
        t_idle = 0;
      }
      s_h = h;
      s_k = k;
      s_sq = sq;
      s_quit = quit;
    }
    __syncthreads();
    const unsigned long long h = s_h;
    const uint32_t k = s_k;
    const uint32_t sq = s_sq;
    const int quit = s_quit;
    __syncthreads();
    if (quit) break;
    if (k == 0) continue;
    // consume one claimed slot per thread
    uint32_t start = 0, deg = 0;
    double delta = 0.0;
    if (threadIdx.x < k) {
      const unsigned long long idx = h + threadIdx.x;
      unsigned long long* slot = self.ring + sq * (self.mask + 1) + (idx & self.mask);
      const unsigned long long want = nb_tag(idx, 0) >> 32;
      unsigned long long x;
      while (((x = ld_acquire(slot)) >> 32) != want) {
        if (nb_aborted(prm.glob)) break;
        __nanosleep(32);
      }
      if ((x >> 32) == want) {
        st_relaxed(slot, 0ull);
        const uint32_t v = (uint32_t)x;
        start = __ldg(self.row_ptr + v);
        deg = __ldg(self.row_ptr + v + 1) - start;
        if (kBfs) {
          // clear the in-queue bit BEFORE reading the depth: a later improvement re-queues (SURVEY 8(a) note 3)
          atom_and_acquire(self.inq + (v >> 5), ~(1u << (v & 31)));
          delta = (double)(ld_relaxed(self.depth + v) + 1u);  // d + 1, exact in f64
        } else {
          // Alg.4: take the residue, add it to the rank, push alpha*rho/deg to the neighbours
          const double rho =
              __longlong_as_double((long long)atomicExch((unsigned long long*)(self.res + v), 0ull));
          if (rho != 0.0) red_add_f64(self.rank + v, rho);
          if (rho == 0.0) deg = 0;  // dangling (deg 0) absorbs (R-PR-3)
          else if (deg) delta = prm.alpha * rho / (double)deg;
        }
      }
    }
    // CTA-level load-balanced expand: block scan of the k degrees, then thread t takes edge
    // e = base + u*kNbBlock + t of the batch's concatenated rows and finds its item by binary search
    uint32_t incl = deg;
    for (int o = 1; o < 32; o <<= 1) {
      const uint32_t y = __shfl_up_sync(0xffffffffu, incl, o);
      if ((int)lane >= o) incl += y;
    }
    if (lane == 31) s_wsum[wid] = incl;
    __syncthreads();
    uint32_t wbase = 0, total = 0;
#pragma unroll
    for (int w2 = 0; w2 < kNbBlock / 32; ++w2) {
      const uint32_t x = s_wsum[w2];
      if (w2 < (int)wid) wbase += x;
      total += x;
    }
    s_off[threadIdx.x] = wbase + incl - deg;
    s_start[threadIdx.x] = start;
    s_delta[threadIdx.x] = delta;
    __syncthreads();
    for (uint32_t base = 0; base < total; base += kNbBlock * kNbU) {
      bool act[kNbU];
      uint32_t o[kNbU], lw[kNbU];
#pragma unroll
      for (int u = 0; u < kNbU; ++u) {
        const uint32_t e = base + u * kNbBlock + threadIdx.x;
        act[u] = false;
        o[u] = 0;
        lw[u] = 0;
        if (e < total) {
          uint32_t j = 0;  // largest j with s_off[j] <= e
#pragma unroll
          for (uint32_t step = kNbBlock / 2; step; step >>= 1)
            if (s_off[j + step] <= e) j += step;
          const uint32_t w = __ldg(self.col + s_start[j] + (e - s_off[j]));
          const double xj = s_delta[j];
          o[u] = prm.shift >= 0 ? (w >> prm.shift) : w / prm.B;
          lw[u] = w - o[u] * prm.B;
          if (kBfs) {
            // Alg.2: atomicMin(depth[w], d+1), activate on improvement; stale-read prefilter
            const uint32_t nd = (uint32_t)xj;
            const NbPeer* pe = prm.peers + o[u];
            if (ld_relaxed(pe->depth + lw[u]) > nd) {
              const uint32_t old = atomicMin(pe->depth + lw[u], nd);
              if (old > nd) {
                const uint32_t bit = 1u << (lw[u] & 31);
                act[u] = !(atom_or_release(pe->inq + (lw[u] >> 5), bit) & bit);
              }
            }
          } else {
            const double old = atomicAdd(prm.peers[o[u]].res + lw[u], xj);
            act[u] = old <= prm.eps && old + xj > prm.eps;  // crossing activation (R-PR-7)
          }
          ++edges;
        }
      }
#pragma unroll
      for (int u = 0; u < kNbU; ++u) {
        if (base + u * kNbBlock < total) nb_push(prm, act[u], o[u], lw[u]);
      }
    }
    __syncthreads();
    // every push of these k items reserved its tail slot before this increment (release)
    if (threadIdx.x == 0) {
      __threadfence();
      atom_add_release(&self.ctl[sq].done, (unsigned long long)k);
    }
  }
  for (int o = 16; o; o >>= 1) edges += __shfl_xor_sync(0xffffffffu, edges, o);
  if (lane == 0 && edges) atomicAdd(&prm.glob->edges, edges);
}

// rank_out = rank / n_global (R-PR-4); residual sum into *sum.
__global__ void k_nb_finalize(NbParams prm, double n_global, double* sum) {
  double acc = 0.0;
  const uint32_t p0 = prm.self < 0 ? 0u : (uint32_t)prm.self, p1 = prm.self < 0 ? prm.P : p0 + 1;
  for (uint32_t p = p0; p < p1; ++p) {
    const NbPeer pe = prm.peers[p];
    for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < pe.n_local;
         v += (int64_t)gridDim.x * blockDim.x) {
      pe.rank[v] = pe.rank[v] / n_global;
      acc += pe.res[v];
    }
  }
  for (int o = 16; o; o >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, o);
  if (lane_id() == 0 && acc != 0.0) atomicAdd(sum, acc);
}

static inline uint64_t nb_pow2(uint64_t x) {
  uint64_t c = 1;
  while (c < x) c <<= 1;
  return c;
}

// BFS source seed: depth[src] = 0, its in-queue bit set, one push into its owner's ring.
__global__ void k_nb_bfs_seed(NbParams prm, uint32_t o, uint32_t l) {
  if (lane_id() == 0) {
    prm.peers[o].depth[l] = 0u;
    prm.peers[o].inq[l >> 5] = 1u << (l & 31);
  }
  __syncwarp();
  nb_push(prm, lane_id() == 0, o, l);
}

// ---------------------------------------------------------------- across processes
// One partition per process (torchrun / the host transport).  Each rank keeps its peer-visible state in
// ONE cudaMalloc block -- its S rings, their counters, its residue (PageRank) or depth words (BFS), its
// in-queue bits, and a global word block -- exported once with a CUDA IPC handle; the handles are
// all-gathered over the communicator and every peer block is mapped (cudaIpcOpenMemHandle, lazy peer
// access: NVLink peer memory across GPUs, the same memory on one GPU).  The kernel is the loopback one:
// this process's CTAs serve only its own sub-queues, and a remote relaxation is an atomic on the owner's
// block plus, on activation, a push into the owner's ring.  Termination is the same global quiescence,
// read over every rank's counters.  Host barriers (allreduce) separate the phases that write another
// rank's memory: init -> (PageRank) init residues -> seeds -> kernels -> end (no rank frees or reuses its
// block while a peer's kernel may still read its counters).
struct NbLayout {
  size_t ring, ctl, state, inq, glob, total;
};
static NbLayout nb_layout(int64_t n_local, uint32_t S) {
  auto al = [](size_t x) { return (x + 255) / 256 * 256; };
  NbLayout L;
  const uint64_t cap = nb_pow2((uint64_t)std::max<int64_t>(n_local, 1024));
  L.ring = 0;
  L.ctl = al(L.ring + (size_t)S * cap * 8);
  L.state = al(L.ctl + (size_t)S * sizeof(NbCtl));
  L.inq = al(L.state + (size_t)std::max<int64_t>(n_local, 1) * 8);
  L.glob = al(L.inq + ((size_t)n_local / 32 + 1) * 4);
  L.total = al(L.glob + sizeof(NbGlob) + 8);
  return L;
}

static int nb_barrier(atos_csr* g, cudaStream_t s) {
  ATOS_CUDA(cudaStreamSynchronize(s));
  uint64_t z = 0;
  return allreduce_u64(g->comm, &z, s);
}

static int run_nobarrier_mp(atos_csr* g, bool bfs, double alpha, double eps, double* rank_out, uint32_t* depth_out,
                            int64_t src, const Resolved& r, atos_stats* st) {
  cudaStream_t s = r.stream;
  const uint32_t P = (uint32_t)g->nranks, me = (uint32_t)g->rank;
  if (P > kNbMaxParts) {
    set_error("barrier_free: at most %u ranks (got %u)", kNbMaxParts, P);
    return ATOS_ERR_UNSUPPORTED;
  }
  if (!bfs && r.check_size > 0) {
    set_error("barrier_free: check_size sweeps are single-partition only");
    return ATOS_ERR_UNSUPPORTED;
  }
  uint32_t S = bfs ? 4u : (P >= 4 ? 1u : 2u);
  if (const char* e = getenv("ATOS_NB_SUBQ")) S = (uint32_t)std::max(1, std::min(16, atoi(e)));
  const uint32_t B = (uint32_t)((g->n + P - 1) / P);
  Part& p = g->parts[0];
  std::vector<int64_t> nl(P);
  for (uint32_t i = 0; i < P; ++i) {
    int64_t b = 0, e = 0;
    atos_partition_range(g->n, (int)P, (int)i, &b, &e);
    nl[i] = e - b;
  }
  const NbLayout mine = nb_layout(nl[me], S);
  // 1. the peer-visible block and the peers' mappings (once per handle)
  if (!p.nb_ipc) {
    ATOS_CUDA(cudaMalloc(&p.nb_ipc, mine.total));
    p.nb_ipc_bytes = mine.total;
    cudaIpcMemHandle_t h;
    ATOS_CUDA(cudaIpcGetMemHandle(&h, p.nb_ipc));
    std::vector<cudaIpcMemHandle_t> all(P);
    ATOS_TRY(allgather_host(g->comm, &h, sizeof(h), all.data(), s));
    p.nb_peer_base.assign(P, nullptr);
    for (uint32_t i = 0; i < P; ++i) {
      if (i == me) continue;
      ATOS_CUDA(cudaIpcOpenMemHandle(&p.nb_peer_base[i], all[i], cudaIpcMemLazyEnablePeerAccess));
    }
  }
  std::vector<NbPeer> peers(P);
  for (uint32_t i = 0; i < P; ++i) {
    char* b = i == me ? (char*)p.nb_ipc : (char*)p.nb_peer_base[i];
    const NbLayout L = nb_layout(nl[i], S);
    const uint64_t cap = nb_pow2((uint64_t)std::max<int64_t>(nl[i], 1024));
    peers[i] = NbPeer{i == me ? p.row_ptr : nullptr, i == me ? p.col : nullptr,
                      (!bfs && i == me) ? rank_out : nullptr, bfs ? nullptr : (double*)(b + L.state),
                      (unsigned long long*)(b + L.ring), (NbCtl*)(b + L.ctl), cap - 1, (uint32_t)nl[i], 0,
                      bfs ? (uint32_t*)(b + L.state) : nullptr, (uint32_t*)(b + L.inq)};
  }
  const size_t tbl = sizeof(NbPeer) * P;
  ATOS_TRY(p.nb_peers.ensure(tbl));
  ATOS_CUDA(cudaMemcpyAsync(p.nb_peers.p, peers.data(), tbl, cudaMemcpyHostToDevice, s));
  char* own = (char*)p.nb_ipc;
  NbGlob* glob = (NbGlob*)((char*)(me == 0 ? p.nb_ipc : p.nb_peer_base[0]) + nb_layout(nl[0], S).glob);
  double* sum = (double*)(own + mine.glob + sizeof(NbGlob));
  int shift = -1;
  if ((B & (B - 1)) == 0) {
    shift = 0;
    while ((1u << shift) < B) ++shift;
  }
  NbParams prm{(const NbPeer*)p.nb_peers.p, glob, P, B, shift, S, alpha, eps, r.watchdog_ns,
                r.timeout_s > 0 ? (unsigned long long)(r.timeout_s * 1e9) : 0ull, (int)me};
  const int gs = 148 * 8;
  // 2. own state (rings, counters, global words, residue / depth, in-queue bits), then a barrier
  ATOS_CUDA(cudaMemsetAsync(own + mine.ring, 0, mine.state - mine.ring, s));
  ATOS_CUDA(cudaMemsetAsync(own + mine.inq, 0, mine.total - mine.inq, s));
  if (bfs) {
    ATOS_CUDA(cudaMemsetAsync(own + mine.state, 0xFF, (size_t)std::max<int64_t>(nl[me], 1) * 4, s));
  } else {
    k_nb_init_vertices<<<gs, 256, 0, s>>>(prm, 1.0 - alpha);
    ++g_launches;
  }
  ATOS_CUDA(cudaGetLastError());
  ATOS_TRY(nb_barrier(g, s));
  // 3. PageRank: every rank's rows add their initial mass into the owners' residues; then a barrier
  if (!bfs) {
    if (nl[me]) {
      k_nb_init_edges<<<gs, 256, 0, s>>>(prm, me, (1.0 - alpha) * alpha);
      ++g_launches;
    }
    ATOS_TRY(nb_barrier(g, s));
  }
  // 4. seeds (own ring), then a barrier: no kernel may observe quiescence before every seed is queued
  if (bfs) {
    if (src >= (int64_t)me * B && src < (int64_t)me * B + nl[me]) {
      k_nb_bfs_seed<<<1, 32, 0, s>>>(prm, me, (uint32_t)(src - (int64_t)me * B));
      ++g_launches;
    }
  } else if (nl[me]) {
    k_nb_seed<<<gs, 256, 0, s>>>(prm, me);
    ++g_launches;
  }
  ATOS_CUDA(cudaGetLastError());
  ATOS_TRY(nb_barrier(g, s));
  // 5. the persistent kernel of this rank
  int grid = 0;
  const void* fn = bfs ? (const void*)k_nobarrier<true> : (const void*)k_nobarrier<false>;
  ATOS_TRY(persistent_grid(fn, kNbBlock, 0, &grid));
  if (r.num_blocks > 0) grid = std::min(grid, r.num_blocks);
  grid = std::max<int>((int)S, grid - grid % (int)S);
  WorkerTimer wt;
  wt.start(s);
  void* args[] = {(void*)&prm};
  ATOS_CUDA(cudaLaunchCooperativeKernel(fn, grid, kNbBlock, args, 0, s));
  ++g_launches;
  wt.stop(s);
  if (stream_wait(s, r.timeout_s) == ATOS_ERR_TIMEOUT) ATOS_CUDA(cudaStreamSynchronize(s));
  // 6. every kernel has stopped before anyone reads results or reuses its block
  ATOS_TRY(nb_barrier(g, s));
  NbGlob hg{};
  ATOS_CUDA(cudaMemcpy(&hg, glob, sizeof(NbGlob), cudaMemcpyDeviceToHost));
  if (hg.abort) {
    set_error("barrier_free %s: %s", bfs ? "BFS" : "PageRank",
              hg.abort == 2 ? "timeout_s exceeded" : "no progress (watchdog)");
    return ATOS_ERR_TIMEOUT;
  }
  double hsum = 0.0;
  if (bfs) {
    if (nl[me]) ATOS_CUDA(cudaMemcpyAsync(depth_out, own + mine.state, (size_t)nl[me] * 4, cudaMemcpyDeviceToDevice, s));
  } else {
    ATOS_CUDA(cudaMemsetAsync(sum, 0, 8, s));
    k_nb_finalize<<<gs, 256, 0, s>>>(prm, (double)g->n, sum);
    ++g_launches;
    ATOS_CUDA(cudaMemcpyAsync(&hsum, sum, 8, cudaMemcpyDeviceToHost, s));
  }
  ATOS_CUDA(cudaStreamSynchronize(s));
  if (!bfs) ATOS_TRY(allreduce_f64(g->comm, &hsum, s));
  if (st) {
    std::vector<NbCtl> hc(S);
    ATOS_CUDA(cudaMemcpy(hc.data(), own + mine.ctl, S * sizeof(NbCtl), cudaMemcpyDeviceToHost));
    for (uint32_t j = 0; j < S; ++j) {
      st->pops += hc[j].done;
      st->pushes += hc[j].tail;
    }
    st->edges += hg.edges;  // every rank's edge visits (the counter is global)
    st->rounds += 1;
    if (!bfs) st->residual_sum = hsum;
    st->worker_ms += wt.elapsed();
  }
  return ATOS_OK;
}

// Shared driver: PageRank (rank_out) or BFS (depth_out, src).
static int run_nobarrier(atos_csr* g, bool bfs, double alpha, double eps, double* rank_out, uint32_t* depth_out,
                         int64_t src, const Resolved& r, atos_stats* st) {
  cudaStream_t s = r.stream;
  if (r.knobs_set) {
    set_error("barrier_free: persistent=0, dedupe=0, worker, fetch_size, queue_capacity, depth_state and "
              "engine_variant do not apply to the barrier-free kernel (its worker is fixed, DESIGN.md section 7)");
    return ATOS_ERR_UNSUPPORTED;
  }
  if (g->comm) return run_nobarrier_mp(g, bfs, alpha, eps, rank_out, depth_out, src, r, st);
  const uint32_t P = (uint32_t)g->num_parts;
  if (P < 2 || P > kNbMaxParts) {
    set_error("barrier_free: needs a loopback-partitioned graph with 2..%u partitions (got %u)", kNbMaxParts, P);
    return ATOS_ERR_UNSUPPORTED;
  }
  if (!bfs && r.check_size > 0) {
    set_error("barrier_free: check_size sweeps are single-partition only");
    return ATOS_ERR_UNSUPPORTED;
  }
  const uint32_t B = (uint32_t)((g->n + P - 1) / P);
  // sub-queues per partition (fewer CTAs per head CAS, but shorter FIFOs pop vertices with less
  // accumulated residue, i.e. more pops); ATOS_NB_SUBQ overrides (tools/nb_ab.py)
  // measured (tools/nb_ab.py, profiles/r01_nobarrier_*subq*): PageRank C3 best at S = 2 for P = 2 and S = 1 for
  // P >= 4 (more sub-queues add pops); BFS C5 best at S = 4 for every P (P=2 82 -> 52 ms, no added work)
  uint32_t S = bfs ? 4u : (P >= 4 ? 1u : 2u);
  if (const char* e = getenv("ATOS_NB_SUBQ")) S = (uint32_t)std::max(1, std::min(16, atoi(e)));
  std::vector<NbPeer> peers(P);
  for (uint32_t i = 0; i < P; ++i) {
    Part& p = g->parts[i];
    if (p.v_begin != std::min<int64_t>(g->n, (int64_t)i * B)) {  // trailing partitions may be empty
      set_error("barrier_free: partition %u does not start at %u * ceil(n/P)", i, i);
      return ATOS_ERR_INVALID_ARG;
    }
    // The in-queue bit (BFS) / crossing rule (PageRank) keep at most one entry per vertex outstanding across
    // a partition's sub-queues, so tail - head <= n_local per ring and n_local slots never lap an unconsumed one.
    const uint64_t cap = nb_pow2((uint64_t)std::max<int64_t>(p.n_local, 1024));
    ATOS_TRY(p.nb_ring.ensure(S * cap * 8));
    ATOS_TRY(p.nb_ctl.ensure(S * sizeof(NbCtl)));
    ATOS_TRY(p.vbuf_a.ensure((size_t)std::max<int64_t>(p.n_local, 1) * 8));  // PR residue / BFS in-queue bits
    ATOS_CUDA(cudaMemsetAsync(p.nb_ring.p, 0, S * cap * 8, s));
    ATOS_CUDA(cudaMemsetAsync(p.nb_ctl.p, 0, S * sizeof(NbCtl), s));
    p.ring_clean = false;  // conservative: the exchange-round path re-clears its own ring anyway
    peers[i] = NbPeer{p.row_ptr, p.col, bfs ? nullptr : rank_out + p.v_begin, bfs ? nullptr : p.vbuf_a.as<double>(),
                      p.nb_ring.as<unsigned long long>(), p.nb_ctl.as<NbCtl>(), cap - 1, (uint32_t)p.n_local, 0,
                      bfs ? depth_out + p.v_begin : nullptr, bfs ? p.vbuf_a.as<uint32_t>() : nullptr};
    if (bfs) {
      // Alg.1 init P:721-725: depth = MAX_UINT32, nothing queued
      if (p.n_local) ATOS_CUDA(cudaMemsetAsync(depth_out + p.v_begin, 0xFF, (size_t)p.n_local * 4, s));
      ATOS_CUDA(cudaMemsetAsync(p.vbuf_a.p, 0, ((size_t)p.n_local / 32 + 1) * 4, s));
    }
  }
  Part& p0 = g->parts[0];
  const size_t tbl = sizeof(NbPeer) * P;
  ATOS_TRY(p0.nb_peers.ensure(tbl + sizeof(NbGlob) + 64));
  char* base = p0.nb_peers.as<char>();
  ATOS_CUDA(cudaMemcpyAsync(base, peers.data(), tbl, cudaMemcpyHostToDevice, s));
  NbGlob* glob = (NbGlob*)(base + tbl);
  double* sum = (double*)(base + tbl + sizeof(NbGlob));
  ATOS_CUDA(cudaMemsetAsync(glob, 0, sizeof(NbGlob) + 8, s));
  int shift = -1;
  if ((B & (B - 1)) == 0) {
    shift = 0;
    while ((1u << shift) < B) ++shift;
  }
  NbParams prm{(const NbPeer*)base, glob, P, B, shift, S, alpha, eps, r.watchdog_ns,
                r.timeout_s > 0 ? (unsigned long long)(r.timeout_s * 1e9) : 0ull, -1};
  const int gs = 148 * 8;
  if (bfs) {
    const uint32_t o = (uint32_t)(src / B);
    k_nb_bfs_seed<<<1, 32, 0, s>>>(prm, o, (uint32_t)(src - (int64_t)o * B));
    ++g_launches;
  } else {
    k_nb_init_vertices<<<gs, 256, 0, s>>>(prm, 1.0 - alpha);
    ++g_launches;
    for (uint32_t i = 0; i < P; ++i) {
      if (g->parts[i].n_local == 0) continue;
      k_nb_init_edges<<<gs, 256, 0, s>>>(prm, i, (1.0 - alpha) * alpha);
      ++g_launches;
    }
    for (uint32_t i = 0; i < P; ++i) {
      if (g->parts[i].n_local == 0) continue;
      k_nb_seed<<<gs, 256, 0, s>>>(prm, i);
      ++g_launches;
    }
  }
  ATOS_CUDA(cudaGetLastError());
  int grid = 0;
  const void* fn = bfs ? (const void*)k_nobarrier<true> : (const void*)k_nobarrier<false>;
  ATOS_TRY(persistent_grid(fn, kNbBlock, 0, &grid));
  if (r.num_blocks > 0) grid = std::min(grid, r.num_blocks);
  const int Q = (int)(P * S);
  grid = std::max<int>(Q, grid - grid % Q);  // every sub-queue gets the same number of CTAs
  WorkerTimer wt;
  wt.start(s);
  void* args[] = {(void*)&prm};
  ATOS_CUDA(cudaLaunchCooperativeKernel(fn, grid, kNbBlock, args, 0, s));
  ++g_launches;
  wt.stop(s);
  if (!bfs) {
    k_nb_finalize<<<gs, 256, 0, s>>>(prm, (double)g->n, sum);
    ++g_launches;
  }
  ATOS_CUDA(cudaGetLastError());
  if (stream_wait(s, r.timeout_s) == ATOS_ERR_TIMEOUT) {
    // the device deadline stops the kernel by itself: wait for it before handing the buffers back
    ATOS_CUDA(cudaStreamSynchronize(s));
  }
  NbGlob hg{};
  double hsum = 0.0;
  ATOS_CUDA(cudaMemcpy(&hg, glob, sizeof(NbGlob), cudaMemcpyDeviceToHost));
  ATOS_CUDA(cudaMemcpy(&hsum, sum, 8, cudaMemcpyDeviceToHost));
  if (hg.abort == 2) {
    set_error("barrier_free %s: timeout_s = %.3f exceeded", bfs ? "BFS" : "PageRank", r.timeout_s);
    return ATOS_ERR_TIMEOUT;
  }
  if (hg.abort) {
    set_error("barrier_free %s: no progress for %.1f s (watchdog)", bfs ? "BFS" : "PageRank", r.watchdog_ns * 1e-9);
    return ATOS_ERR_TIMEOUT;
  }
  if (st) {
    uint64_t pops = 0, pushes = 0;
    for (uint32_t i = 0; i < P; ++i) {
      std::vector<NbCtl> hc(S);
      ATOS_CUDA(cudaMemcpy(hc.data(), g->parts[i].nb_ctl.p, S * sizeof(NbCtl), cudaMemcpyDeviceToHost));
      for (uint32_t j = 0; j < S; ++j) {
        pops += hc[j].done;
        pushes += hc[j].tail;
      }
    }
    st->pops += pops;
    st->pushes += pushes;
    st->edges += hg.edges;
    st->rounds += 1;
    if (!bfs) st->residual_sum = hsum;
    st->worker_ms += wt.elapsed();
  }
  return ATOS_OK;
}


int pagerank_nobarrier(atos_csr* g, double alpha, double eps, double* rank_out, const Resolved& r,
                       atos_stats* st) {
  return run_nobarrier(g, false, alpha, eps, rank_out, nullptr, 0, r, st);
}

int bfs_nobarrier(atos_csr* g, int64_t src, uint32_t* depth_out, const Resolved& r, atos_stats* st) {
  return run_nobarrier(g, true, 0.0, 0.0, nullptr, depth_out, src, r, st);
}

}  // namespace atos
