/*
 * atos.h -- C ABI of the B200-native Atos hot path (libatos.so).
 *
 * Paper: Chen, Brock, Porumbescu, Buluc, Yelick, Owens, "Atos: A Task-Parallel
 * GPU Scheduler for Graph Analytics", ICPP'22 (/root/reference/PAPER.md,
 * cited P:<line>).  The three solver calls follow the paper's problem
 * statements: speculative BFS (Alg.2; Listing 4),
 * asynchronous push PageRank (Alg.3 init + Alg.4) and asynchronous
 * speculative graph colouring (Alg.6).  The scheduler knobs of the
 * paper's Queues API (Listing 3: persistent vs discrete kernel,
 * worker size thread/warp/CTA, FETCH_SIZE, numBlock) are fields of atos_cfg.
 *
 * Conventions (all functions):
 *  - Plain C types only; no exceptions cross the ABI; every call returns an
 *    ATOS_* code (0 = OK) and on failure atos_last_error() returns a
 *    thread-local message.  After an error the output contents are
 *    unspecified.
 *  - Graph: CSR with row_ptr[n+1] (int64, row_ptr[0] = 0, non-decreasing) and
 *    col[m] (int32, 0 <= col < n); row v lists v's out-neighbours.
 *  - Outputs are caller-owned buffers of length n (or the local slice length
 *    for a distributed partition).  cfg->out_where says whether they are
 *    device pointers on the graph's device (default) or host pointers.  The
 *    library never frees caller memory.
 *  - Calls are host-synchronous: they return after the result is complete.
 *    Device work is enqueued on cfg->stream (a cudaStream_t; NULL = the
 *    legacy default stream) so it composes with torch streams.
 *  - A csr handle is internally locked: concurrent solver calls on the same
 *    handle serialise; distinct handles are independent.
 *  - Nothing here reads or writes files, and there is no CPU fallback: a
 *    missing or unusable CUDA device yields ATOS_ERR_CUDA.
 */
#ifndef ATOS_H
#define ATOS_H

#include <stddef.h>
#include <stdint.h>

#if defined(__GNUC__)
#define ATOS_API __attribute__((visibility("default")))
#else
#define ATOS_API
#endif

#ifdef __cplusplus
extern "C" {
#endif

#define ATOS_VERSION 1

/* return codes */
#define ATOS_OK                  0
#define ATOS_ERR_INVALID_ARG    -1  /* null pointer, src out of range, alpha not in (0,1), eps <= 0, bad knob */
#define ATOS_ERR_OOM            -2  /* device or host allocation failed */
#define ATOS_ERR_CUDA           -3  /* CUDA runtime error (incl. no device) */
#define ATOS_ERR_NCCL           -4  /* NCCL error in a distributed call */
#define ATOS_ERR_QUEUE_OVERFLOW -5  /* ring full beyond the watchdog budget */
#define ATOS_ERR_TIMEOUT        -6  /* watchdog / cfg.timeout_s exceeded */
#define ATOS_ERR_NOT_SYMMETRIC  -7  /* atos_color on a non-symmetric CSR (checked when cfg.validate) */
#define ATOS_ERR_UNSUPPORTED    -8  /* e.g. atos_color on a partitioned graph, m >= 2^32 */

/* where a caller buffer lives */
#define ATOS_MEM_HOST   0
#define ATOS_MEM_DEVICE 1

/* worker sizes (Listing 3 launchThread / launchWarp / launchCTA) */
#define ATOS_WORKER_THREAD 1
#define ATOS_WORKER_WARP   32
/* any multiple of 32 in [64, 1024] selects a CTA worker of that many threads */

/* unreachable depth (Alg.1 init MAX_UINT32) */
#define ATOS_UNREACHED 0xFFFFFFFFu

typedef struct atos_csr atos_csr;     /* opaque graph handle: device CSR + cached workspaces */
typedef struct atos_comm atos_comm;   /* opaque multi-process communicator (NCCL) */

/* Counters filled when cfg->stats != NULL (work ratios of Table 4). */
typedef struct {
    uint64_t pops;              /* items dequeued and processed (tasks) */
    uint64_t pushes;            /* items enqueued, including the initial frontier */
    uint64_t edges;             /* neighbour-list entries visited (all tasks) */
    uint64_t rounds;            /* discrete: kernel launches; distributed: exchange rounds; persistent: 1 */
    uint64_t bytes_exchanged;   /* distributed: payload bytes sent by this rank */
    double   kernel_ms;         /* device time of the whole call (init + kernels + exchanges), CUDA events */
    double   residual_sum;      /* PageRank: sum of residues at exit (unnormalised), for conservation checks */
    int64_t  colors_used;       /* colouring: max colour + 1 */
    double   worker_ms;         /* device time of the worker kernel(s) alone (persistent launch, or the sum
                                   of the discrete launches incl. their host round trips), CUDA events */
    uint64_t timeline_len;      /* samples written to cfg->timeline */
    uint64_t flags;             /* bit 0: BFS re-ran with the u32 depth state (depth >= 126 met); bit 1: BFS started
                                   with the u32 state because an earlier call on this graph met depth >= 126 */
    uint64_t max_queue_occupancy; /* largest number of published-but-unclaimed items (tail - head) any worker
                                   saw at a claim (persistent runs; discrete: the largest frontier) */
} atos_stats;

typedef struct {
    uint32_t struct_size;       /* = sizeof(atos_cfg); set by atos_cfg_default */
    int      persistent;        /* 1 persistent kernel (default), 0 discrete per-frontier launches */
    int      worker;            /* 1 thread, 32 warp, 64..1024 CTA; 0 = per-app default (CTA: BFS 256, PageRank 512,
                                   colouring 1024) */
    int      fetch_size;        /* items per pop per worker (FETCH_SIZE); 0 = default (CTA: worker size
                                   for BFS, min(worker,256) for PageRank, min(worker,48) for colouring; warp 8;
                                   thread 1) */
    int      num_blocks;        /* 0 = occupancy max (persistent) / proportional to the frontier (discrete) */
    int      block_threads;     /* threads per block for thread/warp workers; 0 = 256 */
    int      dedupe;            /* 1 (default): in-queue bitmap, a vertex is queued at most once at a time;
                                   0: paper-literal push on every improvement */
    int      check_size;        /* PageRank: 0 = threshold-crossing activation (default);
                                   >0 = the paper's round-robin Check_Size sweep */
    int      conflict_policy;   /* colouring: 0 = the lower-priority endpoint is recoloured (default;
                                   priority = degree, then splitmix64(seed ^ v), then id);
                                   1 = paper-literal, the checker re-queues itself;
                                   2 = as 0 with the hash priority only (no degree term) */
    int      permute_init;      /* colouring: 1 = seed-permuted initial queue order; 0 = vertex-ID order */
    int      validate;          /* 1: check CSR invariants / symmetry at call time (O(m)) */
    int      out_where;         /* ATOS_MEM_DEVICE (default) or ATOS_MEM_HOST for the output buffer */
    uint64_t queue_capacity;    /* ring slots; 0 = auto (power of two >= 2n) */
    double   timeout_s;         /* 0 = none; else the call fails with ATOS_ERR_TIMEOUT */
    void*    stream;            /* cudaStream_t; NULL = legacy default stream */
    atos_stats* stats;          /* optional out */
    int      l2_persist;        /* 1: L2 persisting access-policy window on the hot per-vertex state (BFS state
                                   bytes / depth words, PageRank residue).  The queue counters always carry
                                   per-access L2 evict_last hints (createpolicy), independent of this knob */
    int      big_threshold;     /* persistent CTA/warp workers: a popped vertex with more edges than this is
                                   split into chunks any worker may claim (hub assist); 0 = auto, <0 = off */
    int      big_chunk;         /* edges per hub-assist chunk; 0 = auto */
    uint32_t timeline_cap;      /* samples available in `timeline` (0 = no timeline) */
    uint64_t* timeline;         /* optional DEVICE buffer of 4*timeline_cap uint64: progress samples
                                   (globaltimer ns, tasks done, queue tail, queue head) taken by the
                                   workers every timeline_interval_ns -- the throughput-vs-time data of
                                   the paper's Figs. 1-3 */
    uint32_t timeline_interval_ns; /* 0 = 5000 */
    int      depth_state;       /* BFS state (dedupe mode): 0 = auto -- one byte per vertex (7-bit depth + queued
                                   flag, L2-resident), re-run with u32 words if a depth >= 126 is met;
                                   2 = u32 words from the start (high-diameter graphs) */
    int      engine_variant;    /* BFS/PageRank worker build: 0 = auto (persistent 256-thread CTA workers run the
                                   48-register, 5-CTAs-per-SM build with 2 edges in flight per thread on
                                   graphs with m < 8n and 4 otherwise); 1 = the 64-register build (4 edges
                                   in flight) for every worker size */
    int      barrier_free;      /* BFS / PageRank on a loopback-partitioned graph (num_parts 2..8): 1 = the
                                   barrier-free protocol (NEXT-4, nobarrier.cu): one persistent kernel; a remote
                                   relaxation (BFS atomicMin on depth, PageRank atomicAdd on residue) and its
                                   activation go straight into the owner's slice and queue; global quiescence
                                   termination; 0 (default) = exchange rounds.  ATOS_ERR_UNSUPPORTED on a
                                   single-partition or multi-process graph, and when persistent=0, dedupe=0,
                                   worker, fetch_size, queue_capacity, depth_state or engine_variant is set (the
                                   barrier-free kernel has its own fixed CTA worker); timeout_s is a device
                                   deadline (the kernel stops itself before the call returns ATOS_ERR_TIMEOUT) */
    int      recolor_spread;    /* colouring, CTA worker: 0/1 (default) = every assign takes the smallest free
                                   colour (Alg.6 find_min_color); k > 1 = the a-th RECOLOUR of a
                                   vertex takes the j-th smallest free colour <= deg(v), j = hash mod
                                   min(2^(a-1), k) -- breaks repeated collisions in dense cores at the price
                                   of more colours (DESIGN.md R-GC-10) */
} atos_cfg;

/* Fill *cfg with defaults (persistent, app-default worker/fetch, dedupe on). */
ATOS_API void atos_cfg_default(atos_cfg* cfg);

/*
 * Create a graph handle on CUDA device `device` from a CSR in host or device
 * memory (`where` = ATOS_MEM_HOST / ATOS_MEM_DEVICE).  The library copies the
 * CSR (narrowing offsets to 32 bits; m must be < 2^32, else
 * ATOS_ERR_UNSUPPORTED) and never keeps the caller's pointers.
 * num_parts = 1: ordinary single-GPU graph.  num_parts > 1: the graph is
 * 1D-vertex-block partitioned into num_parts partitions on the SAME device and
 * atos_bfs / atos_pagerank run the multi-GPU exchange protocol with an
 * in-process loopback exchange (a correctness/analysis mode for the
 * distributed path on one GPU).  Invalid CSR (row_ptr not monotone, col out
 * of range) is rejected when it is host memory; device-resident input is
 * checked on the device.
 */
ATOS_API int atos_csr_create(atos_csr** out, int64_t n, int64_t m, const int64_t* row_ptr,
                    const int32_t* col, int where, int device, int num_parts);

/*
 * atos_csr_create with layout flags.  atos_csr_create(...) == atos_csr_create_ex(..., 0).
 *   ATOS_LAYOUT_DEGREE: a single-partition graph is stored in the DEGREE LAYOUT -- vertices relabelled
 *     once, at creation, by descending degree -- so the hubs' per-vertex state is
 *     a compact L2-resident prefix (single-partition PageRank additionally spreads its residue / rank
 *     arrays so that each of the 65536 hottest vertices owns a 128-byte line).  Invisible to the caller: sources are mapped in, outputs are written in the
 *     caller's vertex ids, colouring seeds its queue in the caller's id order.  Costs two u32[n] maps
 *     on the device and one output scatter per call.
 *   ATOS_LAYOUT_AUTO (0): the degree layout when it pays -- an f64 per-vertex array would not fit half
 *     of L2 (n * 8 > L2 / 2) and the degrees are skewed (max degree >= 32 * max(1, m / n)); else input.
 *   ATOS_LAYOUT_INPUT: keep the caller's vertex ids.
 * Partitioned graphs (num_parts > 1) always keep the input ids.
 */
#define ATOS_LAYOUT_AUTO 0
#define ATOS_LAYOUT_INPUT 1
#define ATOS_LAYOUT_DEGREE 2
ATOS_API int atos_csr_create_ex(atos_csr** out, int64_t n, int64_t m, const int64_t* row_ptr,
                                const int32_t* col, int where, int device, int num_parts, int flags);

/* Release a handle and all its device memory.  NULL is a no-op. */
ATOS_API void atos_csr_destroy(atos_csr* g);

/* Query n, m and the number of partitions of a handle (any pointer may be NULL). */
ATOS_API int atos_csr_info(const atos_csr* g, int64_t* n, int64_t* m, int* num_parts);

/* The layout a handle actually uses (ATOS_LAYOUT_INPUT or ATOS_LAYOUT_DEGREE; AUTO is resolved at creation). */
ATOS_API int atos_csr_layout(const atos_csr* g, int* layout);

/*
 * Speculative (asynchronous) BFS from `src` (Alg.2): depth_out[v]
 * = hop distance from src along out-edges, ATOS_UNREACHED if unreachable.
 * Result is exact (bit-identical to a serial BFS) for every schedule.
 * For a distributed partition `src` is a GLOBAL id and depth_out is the local
 * slice [v_begin, v_end).
 */
ATOS_API int atos_bfs(const atos_csr* g, int64_t src, uint32_t* depth_out, const atos_cfg* cfg);

/*
 * Asynchronous push PageRank (Alg.3 init, Alg.4 loop) with damping
 * alpha (the paper's lambda) and residue threshold eps (unnormalised):
 * rank_out[v] = x_v / n where x approximates x = (1-alpha)1 + alpha P^T x
 * with 0 <= x* - x <= eps x* / (1-alpha) elementwise.  fp64 throughout.
 */
ATOS_API int atos_pagerank(const atos_csr* g, double alpha, double eps, double* rank_out,
                  const atos_cfg* cfg);

/*
 * Asynchronous speculative greedy colouring (Alg.6; uberkernel,
 * P:707-717): color_out[v] >= 0, color_out[u] != color_out[w] for every edge
 * u != w, color_out[v] <= deg(v).  `seed` sets the recolouring priority
 * splitmix64(seed ^ v) and the permute_init order.  Requires a symmetric CSR;
 * single partition only (ATOS_ERR_UNSUPPORTED otherwise).
 */
ATOS_API int atos_color(const atos_csr* g, uint64_t seed, int32_t* color_out, const atos_cfg* cfg);

/* ---- bulk-synchronous baselines (the paper's comparison point) ----------- */
/*
 * The BSP versions of the three applications, run on the same handle and
 * with the same result conventions, so Atos can be compared against BSP on
 * the same device (the paper's Table 1 comparison):
 *  - atos_bfs_bsp:      Alg.1, level-synchronous; depth_out exact
 *                       (bit-identical to atos_bfs).
 *  - atos_pagerank_bsp: Alg.3: per iteration every frontier
 *                       vertex pushes its whole residue, then the frontier is
 *                       rebuilt as {v : residue[v] > eps}; same init, output
 *                       scale and error bound as atos_pagerank.
 *  - atos_color_bsp:    Alg.5: assign kernel, barrier, conflict
 *                       kernel; a conflict re-queues the lower-priority
 *                       endpoint (priority as atos_color), or both
 *                       endpoints with cfg->conflict_policy = 1 (the literal
 *                       Alg.5, which may not terminate: set timeout_s).
 * Used cfg fields: stream, stats, out_where, timeout_s, validate
 * (colouring), conflict_policy (colouring); the scheduler knobs are ignored.
 * stats: pops = frontier items processed (colouring: assign + check),
 * rounds = iterations (barriers), edges = neighbour entries visited.
 * Single partition only (ATOS_ERR_UNSUPPORTED otherwise).  Each iteration
 * ends with a host round trip reading the next frontier's size (the paper's
 * cudaDeviceSynchronize() barrier).
 */
ATOS_API int atos_bfs_bsp(const atos_csr* g, int64_t src, uint32_t* depth_out, const atos_cfg* cfg);
ATOS_API int atos_pagerank_bsp(const atos_csr* g, double alpha, double eps, double* rank_out,
                               const atos_cfg* cfg);
ATOS_API int atos_color_bsp(const atos_csr* g, uint64_t seed, int32_t* color_out, const atos_cfg* cfg);

/* ---- multi-process (one process per GPU, e.g. torchrun) ------------------ */

#define ATOS_COMM_ID_BYTES 128

/* Write a fresh NCCL unique id (ATOS_COMM_ID_BYTES bytes) to id_out; call on rank 0 and broadcast. */
ATOS_API int atos_comm_unique_id(void* id_out, size_t len);

/* Create the communicator of rank `rank` of `nranks` on CUDA device `device`. Collective. */
ATOS_API int atos_comm_create(atos_comm** out, int nranks, int rank, const void* id, size_t len, int device);
ATOS_API void atos_comm_destroy(atos_comm* comm);

/*
 * Host-staged transport: a communicator whose two exchange steps (per-destination counts, then the
 * SoA payloads of each round) and termination allreduces go through the
 * caller's own host collectives instead of NCCL -- e.g. torch.distributed over gloo or MPI.  Used
 * where NCCL cannot run (several ranks sharing one GPU in tests; no NVLink) and as the reference
 * transport the NCCL path is checked against.  All buffers are HOST memory owned by the library for
 * the duration of the call; the callbacks must be collective (every rank calls them in the same
 * order) and return 0 on success.
 *   alltoallv: rank r sends send_bytes[p] bytes starting at send + sum(send_bytes[0..p)) to rank p
 *              and receives recv_bytes[p] bytes from rank p into recv + sum(recv_bytes[0..p)).
 *   allreduce: in-place sum over ranks of ONE value: dtype 0 = uint64_t, 1 = double.
 */
typedef int (*atos_host_alltoallv_fn)(void* user, const void* send, const uint64_t* send_bytes, void* recv,
                                      const uint64_t* recv_bytes);
typedef int (*atos_host_allreduce_fn)(void* user, void* value, int dtype);
ATOS_API int atos_comm_create_host(atos_comm** out, int nranks, int rank, int device,
                                   atos_host_alltoallv_fn alltoallv, atos_host_allreduce_fn allreduce, void* user);

/*
 * Create this rank's partition of a 1D vertex-block partitioned graph: the
 * rank owns global vertices [v_begin, v_end) and passes their rows
 * (row_ptr_local[v_end-v_begin+1], offsets starting at 0; col_global[m_local]
 * holds GLOBAL vertex ids).  Partitions must tile [0, n_global) in rank order.
 * The handle keeps a reference to `comm` (which must outlive it).
 */
ATOS_API int atos_csr_create_part(atos_csr** out, atos_comm* comm, int64_t n_global, int64_t v_begin,
                         int64_t v_end, int64_t m_local, const int64_t* row_ptr_local,
                         const int32_t* col_global, int where);

/*
 * Gather the ranks' output slices (atos_bfs depth / atos_pagerank rank, device pointers on each rank's
 * device, slice [v_begin, v_end) of atos_partition_range) into ONE array of n_global elements of
 * elem_bytes each on rank 0: out_root is a device pointer on rank 0's device (ignored elsewhere).
 * Collective over the communicator (NCCL point-to-point, or the host transport of
 * atos_comm_create_host); enqueued on `stream` (cudaStream_t, NULL = default) and complete on return.
 * This is the multi-process form of SURVEY 8(b)'s "outputs on the first device".
 */
ATOS_API int atos_comm_gather(atos_comm* comm, int64_t n_global, const void* slice, size_t elem_bytes,
                              void* out_root, void* stream);

/* Block partition used by the library: rank r owns [r*ceil(n/P), min(n,(r+1)*ceil(n/P))). */
ATOS_API int atos_partition_range(int64_t n, int nparts, int part, int64_t* v_begin, int64_t* v_end);

/* ---- misc ---------------------------------------------------------------- */

ATOS_API const char* atos_last_error(void);
ATOS_API int atos_version(void);
/* Number of the library's own kernel launches since load (for launch accounting). */
ATOS_API uint64_t atos_kernel_launches(void);

#ifdef __cplusplus
}
#endif
#endif /* ATOS_H */
