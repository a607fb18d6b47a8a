/*
 * accmg.h — C ABI of the B200-native multi-GPU parallel-loop runtime.
 *
 * What it implements: the data-parallel hot path of Komoda, Miwa, Nakamura, Maruyama,
 * "Integrating Multi-GPU Execution in an OpenACC Compiler" (ICPP'13). Citations "L<n> §<s>"
 * are lines of the paper text and their section. One offloaded `parallel loop` runs in
 * the paper's three BSP steps (L64 §III.A): (1) the iteration space is divided into tasks mapped
 * to GPUs and the data each GPU may read is loaded; (2) every GPU runs its tasks; (3) inter-GPU
 * communication restores coherence, then a global barrier.
 *
 * The paper's translator (L100-114 §IV.B) is replaced by this explicit ABI: loop bodies are
 * hand-written sm_100a kernels selected by `body_id`, and the translator's "array configuration
 * information" (L114) is the `accmg_access` descriptor list passed with every launch.
 *
 * Conventions (all entry points):
 *   - return int status: ACCMG_OK (0) or a negative ACCMG_E* code; no exception crosses the ABI;
 *   - after a CUDA or NCCL failure the error is sticky: every later call returns the same code and
 *     accmg_last_error() describes the first failure;
 *   - not thread-safe: one host thread per process drives the library;
 *   - multi-process (SPMD, one process per GPU, e.g. torchrun): every call except the debug and
 *     stats getters is collective — every rank makes the same calls with the same arguments
 *     (host pointers excepted), in the same order.
 */
#ifndef ACCMG_H
#define ACCMG_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

/* ---- status codes ------------------------------------------------------------------------- */
#define ACCMG_OK            0
#define ACCMG_EINVAL       -1  /* invalid argument (null, bad mode/stride, unknown body, wrong descs) */
#define ACCMG_ECUDA        -2  /* CUDA runtime error (sticky) */
#define ACCMG_ENCCL        -3  /* NCCL error or NCCL unavailable when world_size > 1 (sticky) */
#define ACCMG_ENOMEM       -4  /* device or host allocation failed */
#define ACCMG_ESTATE       -5  /* not initialised / already initialised / region in use / data lost */
#define ACCMG_EUNSUPPORTED -6  /* e.g. more than 64 partitions, shape a body does not support */
#define ACCMG_ECONFLICT    -7  /* debug_checks: overlapping declared writes or two writers of one element */
#define ACCMG_EDATA        -8  /* input violates a body's stated precondition (checked on device) */

/* ---- configuration ------------------------------------------------------------------------ */
/* exchange_mode */
#define ACCMG_XCHG_AUTO     0  /* same-process partitions: device copies / direct scatter;
                                  other processes (P2P): peers' replicas are mapped through CUDA
                                  IPC — pulls are copy-engine reads over NVLink, dirty runs are
                                  pushed by one scatter kernel into every replica, reductions read
                                  all partials; a device-side flag barrier closes each loop */
#define ACCMG_XCHG_NCCL_ALL 1  /* every inter-partition move goes through NCCL, even between
                                  partitions of one process (self send/recv) — for testing */
#define ACCMG_XCHG_NCCL     2  /* across processes: NCCL send/recv and all-reduce */

/* dirty_protocol */
#define ACCMG_DIRTY_RUNS   0
#define ACCMG_DIRTY_CHUNKS 1
/* halo_mode (declared windows) */
#define ACCMG_HALO_AUTO 0      /* push predicted halos from the writing kernel when the body can */
#define ACCMG_HALO_PULL 1      /* the paper's data loader only: pull before read (L119, L125) */

#define ACCMG_MC_OFF  0        /* accmg_config.multicast */
#define ACCMG_MC_AUTO 1
#define ACCMG_MC_VMM  2

typedef struct accmg_config {
    int32_t num_partitions;    /* P, the number of tasks groups every loop is divided into (L108);
                                  1..64; a multiple of world_size. P / world_size partitions live on
                                  each process's GPU ("virtual partitions" when > 1). */
    int32_t world_size;        /* processes (one per GPU); 1 = single process */
    int32_t rank;              /* this process, 0..world_size-1 */
    int32_t device;            /* CUDA device ordinal this process drives; -1 = host-only dry run
                                  (planning and byte accounting without any CUDA call; loop bodies
                                  are not executed) */
    int64_t dirty_chunk_bytes; /* second-level dirty-bit chunk (L135: "we experimentally choose 1MB");
                                  bytes of array data per chunk bit; 0 = 1<<20; a power of two >= 256
                                  (ACCMG_EINVAL otherwise) */
    int32_t exchange_mode;     /* ACCMG_XCHG_* */
    int32_t debug_checks;      /* 1 = check declared-write disjointness (G14) and dirty-set
                                  disjointness (L62), keep per-loop bitmap snapshots for the
                                  debug getters; costs extra device work */
    int32_t profile;           /* 1 = time body / compaction / exchange phases with CUDA events */
    int32_t dirty_protocol;    /* undeclared writes: ACCMG_DIRTY_RUNS (default: compacted maximal runs
                                  in the canonical packed buffer, scattered into the peers) or
                                  ACCMG_DIRTY_CHUNKS (the paper's protocol, L133-135: every dirty
                                  chunk with its first-level bits, merged by the bits; same-node
                                  transports only) */
    int32_t halo_mode;         /* ACCMG_HALO_AUTO (default): when a loop writes a declared window and
                                  another partition's last declared read window of that array
                                  overlaps it (iterative codes reuse their patterns, L125), a body
                                  that supports it (2-D Jacobi) stores those rows into that
                                  partition's replica too (P2P mapping over NVLink, or a local
                                  replica) and the rows count as valid there, so the next reader
                                  pulls nothing; the bytes are accounted as declared transfers.
                                  ACCMG_HALO_PULL: pull-before-read only. */
    int32_t multicast;         /* §8 row f3, P2P mode (world_size > 1, one partition per process):
                                  ACCMG_MC_OFF (default) CUDA-IPC replicas, unicast pushes;
                                  ACCMG_MC_AUTO: replicas of arrays written without a declared
                                  pattern (fp32 / 64-bit elements) are driver-VMM allocations
                                  shared through file descriptors and, where the node can create
                                  an NVLS multicast object (accmg_multicast_probe), bound to one:
                                  the compaction pass stores every dirty element once, through
                                  the multicast address (multimem.st), into all replicas;
                                  otherwise (or ACCMG_MC_VMM) unicast pushes into the shared
                                  VMM replicas. Ignored without the P2P transport. */
    uint8_t nccl_unique_id[128]; /* world_size > 1: the job's id, made on rank 0 by
                                    accmg_nccl_unique_id() (NCCL modes) or accmg_unique_id() (P2P),
                                    broadcast by the caller (e.g. torch.distributed); P2P mode names
                                    its single-node shared-memory bootstrap after it */
} accmg_config;

/* ---- regions (device arrays) --------------------------------------------------------------- */
typedef struct accmg_region_s* accmg_region;  /* opaque, library-owned */

/* ---- loop description ---------------------------------------------------------------------- */
typedef struct accmg_bounds {
    int32_t ndim;              /* 1..3 */
    int32_t pad;
    int64_t lo[3], hi[3];      /* half-open iteration ranges; dim 0 (outermost) is the one divided
                                  among partitions (L108, reading G5) */
} accmg_bounds;

/* access modes of one array in one loop (the translator's array configuration information, L114:
   read-only / write-only / localaccess range / reduction destination) */
#define ACCMG_R          1
#define ACCMG_W          2
#define ACCMG_RW         3
#define ACCMG_REDUCE_SUM 4     /* reductiontoarray destination (L89-91 §III.C): dst[idx] += v with
                                  idx chosen at run time; int64 elements; merged hierarchically
                                  (block, GPU, across GPUs — L112) */

typedef struct accmg_access {
    accmg_region region;
    int32_t mode;              /* ACCMG_R / W / RW / REDUCE_SUM */
    int32_t declared;          /* 1: a localaccess window is given (distribution policy, L121-123);
                                  0: replica policy (L121), writes tracked by dirty bits (L133-135) */
    int64_t stride, left, right; /* declared window of iteration i: elements
                                  [stride*i - left, stride*(i+1) - 1 + right] (L87), clipped to the
                                  region; stride > 0, left, right >= 0. Writes of a declared W/RW
                                  array must stay inside its window (L163) and windows of different
                                  partitions must not overlap (owner computes, reading G14). */
} accmg_access;

/* ---- loop bodies (hand-written sm_100a kernels) ---------------------------------------------
 * Descriptor order and args struct per body; every array is a region of the stated element type.
 *
 * ACCMG_BODY_JACOBI2D_5PT: bounds ndim=2 rows [1,R-1) x cols [1,C-1) (or a sub-box of it);
 *   descs [src R (fp32 R*C), dst W (fp32 R*C)];
 *   dst[i][j] = 0.25f*((src[i-1][j] + src[i+1][j]) + (src[i][j-1] + src[i][j+1])).
 *   Declared form: src stride=C left=C right=C, dst stride=C left=right=0.
 * ACCMG_BODY_GEMM_BF16_F32: bounds ndim=2 [0,M) x [0,N);
 *   descs [A R (bf16 M*K, declared stride=K), B R (bf16 K*N, undeclared), C W (fp32 M*N, declared
 *   stride=N)]; C[i][j] = sum_k A[i][k]*B[k][j], fp32 accumulation on tcgen05 tensor cores.
 *   Shapes: N % 8 == 0 and K % 64 == 0 (else ACCMG_EUNSUPPORTED); any M. The k order of every
 *   element is ascending in blocks of 64 (no split-K), independent of the partition count.
 * ACCMG_BODY_KMEANS_ASSIGN: bounds ndim=1 [0,n);
 *   descs [x R (fp32 n*d, declared stride=d), centroids R (fp32 k*d), member W (int32 n, declared
 *   stride=1), sums REDUCE_SUM (int64 k*d), counts REDUCE_SUM (int64 k)];
 *   member[p] = argmin_c fmaf-chain sum_j (x[p][j]-cen[c][j])^2 (lowest c on ties);
 *   sums[member[p]][j] += x[p][j] * 2^shift (exact int64; x must lie on the 2^-shift grid with
 *   |x * 2^shift| < 2^31, else ACCMG_EDATA); counts[member[p]] += 1.
 *   Exact mode, shift = ACCMG_KMEANS_EXACT (reading KM-X; arbitrary finite fp32 points, d <= 64,
 *   k*d <= 16384): sums is int64 k*d*ACCMG_KMEANS_WINDOWS; the exact real sum of the members'
 *   x[p][j] is kept as sum_w sums[c][j][w] * 2^(32w - 149) (every addend below 2^32 in
 *   magnitude: exact for n < 2^31); a non-finite x gives ACCMG_EDATA.
 * ACCMG_BODY_KMEANS_UPDATE: bounds ndim=1 [0,k);
 *   descs [sums RW (int64 k*d, or k*d*ACCMG_KMEANS_WINDOWS in exact mode), counts RW (int64 k),
 *   centroids W (fp32 k*d)];
 *   if counts[c] > 0: cen[c][j] = (float)(((double)sums[c][j] * 2^-shift) / (double)counts[c]);
 *   exact mode: cen[c][j] = (float)(RN64(exact sum) / (double)counts[c]) (the mean of the members:
 *   the exact sum rounded once to double, PAPER.md L219-226 / L89-91);
 *   then sums[c][*] = 0, counts[c] = 0.
 * ACCMG_BODY_JACOBI2D_DEEP: as ACCMG_BODY_JACOBI2D_5PT but each loop performs h sweeps (deep halos,
 *   §8 row f2): dst = J^h(src) on the bounds box, J the 5-point sweep above, rows/columns outside
 *   the box fixed. Declared form: src stride=C left=right=h*C, dst stride=C — one exchange of h
 *   halo rows per h sweeps; each partition recomputes the rows of its halo (redundant compute) in
 *   scratch buffers. args {rows, cols, h}.
 * ACCMG_BODY_JACOBI3D_7PT: bounds ndim=3 [1,n0-1) x [1,n1-1) x [1,n2-1) (or a sub-box); descs
 *   [src R (fp32 n0*n1*n2), dst W (fp32 n0*n1*n2)]; n2 % 4 == 0;
 *   dst[i][j][k] = ((((u+d) + (n+s)) + ((w+e) + (c+c))) * 0.125f with u/d = src[i-1/i+1][j][k],
 *   n/s = src[i][j-1/j+1][k], w/e = src[i][j][k-1/k+1], c = src[i][j][k] (multi-dimensional
 *   stencil of L256; planes are partitioned: declared src stride=n1*n2 left=right=n1*n2).
 * ACCMG_BODY_SCATTER: bounds ndim=1 [0,n); descs [src R (fp32 n, declared stride=1), idx R (int32 n,
 *   declared stride=1), dst W (fp32 m, declared stride=1)]; dst[idx[i]] = src[i] (irregular writes,
 *   the BFS class: idx[i] may fall outside the writer's window). Every write is checked against the
 *   partition's write window (L137 §IV.D.2); a miss appends (index, value) to the partition's
 *   system buffer, and after the kernel the buffered writes are completed in the owner's replica
 *   (the partition whose window holds the index) — L137, L163. Indices must be distinct (L62) and
 *   lie in some partition's window of dst: a record whose index no window holds (negative, >= m,
 *   or in a gap between windows) is dropped, and the next synchronising call (sync_to_host,
 *   barrier, get_stats) returns ACCMG_EDATA.
 * ACCMG_BODY_TEST_SPARSE_WRITE: bounds ndim=1 rows [0,R); descs [in R (fp32 R*C), out W (fp32 R*C)];
 *   rows i with i % period == 0: out[i][j] = in[i][j] + 1.0f for all j (exercises L2 chunk skipping).
 * ACCMG_BODY_TEST_MASKED_WRITE: bounds ndim=1 [0,n); descs [in R (fp32 n), mask R (uint8 n),
 *   out W (fp32 n)]; out[e] = in[e] + 1.0f where mask[e] != 0 (arbitrary dirty-bit patterns for
 *   the compaction of L133-135: isolated bits, runs across words, tiles and chunks). args {n}.
 */
#define ACCMG_BODY_JACOBI2D_5PT      1
#define ACCMG_BODY_GEMM_BF16_F32     2
#define ACCMG_BODY_KMEANS_ASSIGN     3
#define ACCMG_BODY_KMEANS_UPDATE     4
#define ACCMG_BODY_SCATTER           5
#define ACCMG_BODY_JACOBI3D_7PT      6
#define ACCMG_BODY_JACOBI2D_DEEP     7
#define ACCMG_BODY_TEST_SPARSE_WRITE 100
#define ACCMG_BODY_TEST_MASKED_WRITE 101

typedef struct { int64_t rows, cols; } accmg_args_jacobi2d;
typedef struct { int64_t M, N, K; } accmg_args_gemm;
typedef struct { int64_t n; int32_t d, k, shift, pad; } accmg_args_kmeans;
#define ACCMG_KMEANS_EXACT   (-1) /* accmg_args_kmeans.shift: arbitrary finite points (exact sums) */
#define ACCMG_KMEANS_WINDOWS 9    /* int64 windows per (cluster, dim) of the exact-mode sums */
typedef struct { int64_t rows, cols, period; } accmg_args_sparse;
typedef struct { int64_t n; } accmg_args_masked;
typedef struct { int64_t n, m; } accmg_args_scatter;
typedef struct { int64_t n0, n1, n2; } accmg_args_jacobi3d;
typedef struct { int64_t rows, cols, h; } accmg_args_jacobi2d_deep;

/* ---- statistics (E5-style breakdown, L188; device memory User/System, L249) ------------------
 * Byte counters are this process's: pulls into its partitions (receiver-counted), packets its
 * partitions sent (sender-counted, x (P-1) deliveries) and its V/P share of each reduction. With one
 * process they are the whole job's; with several, the whole job's is the sum over ranks. */
typedef struct accmg_stats {
    int64_t loops;                    /* loop launches */
    int64_t bytes_interpartition;     /* all bytes delivered between partitions (sum of the next 4) */
    int64_t bytes_declared;           /* window/halo pulls between partitions (data loader, L119) */
    int64_t bytes_undeclared_payload; /* dirty element values delivered to peers (L131) */
    int64_t bytes_undeclared_headers; /* size words + run starts/ends delivered to peers */
    int64_t bytes_reduce;             /* reductiontoarray merges: 2(P-1)*extent*esize per loop */
    int64_t bytes_paper_protocol;     /* what whole-chunk + L1-bits transfers (L133-135) would move */
    int64_t bytes_remote;             /* subset of bytes_interpartition that crossed processes */
    int64_t bytes_h2d, bytes_d2h;     /* host<->device (data loader copy-in / copy-out) */
    int64_t body_launches;            /* loop-body kernel launches */
    int64_t kernel_launches;          /* all kernels launched by the library */
    int64_t device_bytes_user;        /* replicas on this process's GPU */
    int64_t device_bytes_system;      /* bitmaps, packed/receive buffers, partials (L249-252) */
    double  ms_body, ms_compact, ms_exchange; /* profile=1: summed CUDA-event times */
    int64_t write_misses;             /* distributed-array writes outside the writer's window (L137) */
    int64_t bytes_write_miss;         /* (index, value) records delivered to owners: 8 + esize each */
    /* Bytes the transport actually moves between partitions' memories (the counters above are the
       algorithmic volumes of reading W8): pulls and pushes as above; dirty elements pushed by the
       compaction pass = payload only (no run headers or sizes); NCCL packets = headers + payload;
       a P2P reductiontoarray reads the P-1 other partials on every process (P(P-1) extent esize
       per loop with one partition per process); an in-process merge reads V-1 partials; a write
       miss stores esize into the owner's replica. */
    int64_t bytes_link;
    int64_t bytes_link_remote;        /* subset of bytes_link that crossed processes (NVLink) */
    int64_t bytes_multicast;          /* dirty payload stored once through NVLS multicast addresses
                                         (the switch delivers it to the other replicas) */
    int64_t multicast_regions;        /* regions whose replicas are bound to a multicast object */
} accmg_stats;

/* ---- entry points ------------------------------------------------------------------------- */

/* Writes a fresh NCCL unique id (128 bytes) for accmg_config.nccl_unique_id. Call on rank 0 only.
   Loads NCCL (libnccl.so.2) on first use. */
int accmg_nccl_unique_id(uint8_t out[128]);

/* Writes 128 random bytes (from /dev/urandom) usable as the P2P-mode job id. Rank 0 only. */
int accmg_unique_id(uint8_t out[128]);

/* Runtime start-up (L104 "control codes to initialize the devices"): selects the device, creates
   the process's stream and (world_size > 1) the NCCL communicator. ACCMG_ESTATE if initialised. */
int accmg_init(const accmg_config* cfg);

/* Frees every region and runtime buffer (and the block cache), destroys the stream and
   communicator. */
int accmg_finalize(void);

/* Data-region entry (copyin semantics, L119 §IV.C). Registers `extent` elements of `elem_size`
   bytes at `host_array` (caller-owned, borrowed until accmg_region_destroy; must stay valid and
   unchanged). Device replicas are allocated lazily and only as large as each partition needs: the
   hull of its declared windows for distributed arrays (L121-123 "only the sub-array actually
   accessed by the GPU is loaded"), the whole array for replicated ones; kernels still use global
   indices (the replica pointer is offset, so the index rewriting of L110 is the identity). Before
   each loop the data loader copies in only what each partition may read and does not yet hold
   (L119, L125). elem_size in {1,2,4,8}. */
int accmg_region_create(void* host_array, size_t elem_size, int64_t extent, accmg_region* out);

/* Data-region exit without copy-out (OpenACC `delete`); frees the region's device memory. In a
   one-process run (world_size 1) the freed blocks stay in the runtime's block cache and serve
   later allocations of the same size (no cudaMalloc / cudaFree per re-created region); the cache
   is emptied when an allocation fails (then retried) and at accmg_finalize. */
int accmg_region_destroy(accmg_region r);

/* One offloaded parallel loop (L64 §III.A): partition dim 0 of `bounds` into P chunks
   (chunk g = [lo + floor(g*n/P), lo + floor((g+1)*n/P)), L108), pull what each partition reads
   (L119), run body `body_id` on every chunk, then restore coherence: declared writes change
   ownership; undeclared writes are tracked with two-level dirty bits, compacted into packed
   runs and scattered into every other replica (L129-135); REDUCE_SUM destinations are merged
   across partitions (L112). Enqueued on the library stream; returns without waiting, except that
   undeclared writes with world_size > 1 synchronise the host once to size the NCCL messages.
   `args` points to the body's args struct (args_bytes = its size). n_descs <= 16. */
int accmg_loop_launch(const accmg_bounds* bounds, int body_id, const accmg_access* descs,
                      int n_descs, const void* args, size_t args_bytes);

/* Copy-out (region exit / `update host`, L119): blocks until this process's host array holds
   the coherent contents of the whole region. */
int accmg_sync_to_host(accmg_region r);

/* Distributed copy-out: this process copies to its host array only the ranges whose lowest-index
   holder partition lives on this process; the union over ranks covers the region. Blocks. */
int accmg_sync_to_host_owned(accmg_region r);

/* Waits for all enqueued loops, exchanges and copies of this process (global barrier, L64). */
int accmg_barrier(void);

/* Statistics since init or the last reset (synchronises to read device-side counters). */
int accmg_get_stats(accmg_stats* out);
int accmg_reset_stats(void);

/* Turns the per-phase CUDA-event timing of accmg_config.profile on (1) or off (0) for the loops
   launched from now on. The events sit between consecutive kernels on the library stream, so they
   also stop a loop body from overlapping its launch with the previous body's tail. */
int accmg_set_profile(int on);

/* §8 row f3: can this node create an NVLS multicast object spanning `num_devices` GPUs (the
   driver VMM entry points present and cuMulticastCreate accepted)? Returns 1 if so; 0 if not,
   with the reason copied into why (NUL-terminated, at most cap bytes; may be NULL); negative on
   an argument error. Needs no accmg_init; initialises the CUDA context of the current device. */
int accmg_multicast_probe(int num_devices, char* why, int cap);

/* Text of the sticky error (or the last argument error); never NULL. */
const char* accmg_last_error(void);

/* The cudaStream_t (as void*) all work of this process is enqueued on; NULL before init. */
void* accmg_stream(void);

/* Partition -> iteration chunk of the last loop's dim 0, computed host-side (no CUDA). */
int accmg_chunk(int64_t lo, int64_t hi, int num_partitions, int partition, int64_t* a, int64_t* b);

/* ---- debug getters (partition must live on the calling process) ---------------------------- */
/* Snapshot of `partition`'s first-level dirty bitmap of `r` as set by the last loop that wrote r
   undeclared (needs debug_checks=1): bit b of word w = element 32w+b. nwords = ceil(extent/32). */
int accmg_debug_dirty_bitmap(accmg_region r, int partition, uint32_t* out_words, int64_t nwords);
/* Same for the second-level chunk bits: ceil(ceil(extent/chunk_elems)/32) words. */
int accmg_debug_chunk_bits(accmg_region r, int partition, uint32_t* out_words, int64_t nwords);
/* The canonical packed buffer `partition` sent for `r` in the last loop that wrote r undeclared:
   uint64 n_runs, uint64 n_elems, int64 run_start[n_runs], int64 run_end[n_runs] (exclusive),
   payload (elem_size * n_elems bytes). *used = its size; copies min(cap, size) bytes. */
int accmg_debug_packed(accmg_region r, int partition, void* out, int64_t cap, int64_t* used);
/* Copies `partition`'s replica into out (an extent * elem_size buffer) at the same offsets; only
   the allocated hull is written and only the valid ranges (accmg_debug_valid) hold defined values.
   Blocks. */
int accmg_debug_replica(accmg_region r, int partition, void* out);
/* Valid intervals [lo, hi) of `partition`'s replica (any partition; host-side table):
   out_pairs receives up to cap pairs, *n the total count. partition = -1: this process's host copy. */
int accmg_debug_valid(accmg_region r, int partition, int64_t* out_pairs, int64_t cap, int64_t* n);

#ifdef __cplusplus
}
#endif
#endif /* ACCMG_H */
