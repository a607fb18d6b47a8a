// Internal launch interface of the sm_100a kernels (no torch types; plain pointers and sizes).
// Every launcher enqueues on `s`, adds the number of kernels it launched to *launches, and
// returns the launch error (cudaSuccess if all launches were accepted).
#pragma once
#include <cstdint>
#include <cuda_runtime_api.h>

namespace accmg {
namespace k {

// Two-level dirty bits of one replica (L133-135): l1 = 1 bit per element (bit b of word w is
// element 32w+b), l2 = 1 bit per chunk of 2^l2_shift elements. l1 == nullptr: no tracking.
struct Track {
    uint32_t* l1;
    uint32_t* l2;
    int l2_shift;
};

// Up to 64 device pointers passed by value in the kernel parameter block (no staging copy).
constexpr int kMaxPtrs = 64;
struct PtrList {
    void* p[kMaxPtrs];
    int n;
    int mc;  // 1: p[0] is an NVLS multicast address (one multimem.st reaches every bound replica)
};

// Predicted-halo push of a row-block body: rows [lo[k], hi[k]) of its output are stored also into
// dst[k] (another partition's replica of the output array, global-index base; a local replica or
// a peer's mapped over NVLink), from the same registers as the local store.
constexpr int kMaxPush = 4;
struct HaloPush {
    float* dst[kMaxPush];
    int64_t lo[kMaxPush], hi[kMaxPush];
    int n;
};

// ---- loop bodies -----------------------------------------------------------------------------
// 5-point Jacobi on rows [r0, r1) x cols [c0, c1) of a rows x cols fp32 array (global indices);
// [src_lo, src_hi) = elements allocated behind src.
// impl 0: TMA-staged shared-memory tiles (jacobi2d_tma.cu) where the shape and alignment allow,
// else the register row-marching kernel (LDG.128 sliding window); impl 1: always the latter.
cudaError_t jacobi2d(const float* src, float* dst, int64_t rows, int64_t cols, int64_t r0, int64_t r1,
                     int64_t c0, int64_t c1, int64_t src_lo, int64_t src_hi, Track t, int impl, cudaStream_t s,
                     int64_t* launches, const HaloPush& push = HaloPush{});
cudaError_t jacobi2d_tma(const float* src, float* dst, int64_t rows, int64_t cols, int64_t r0, int64_t r1, int64_t c0,
                         int64_t c1, int64_t src_lo, int64_t src_hi, Track t, cudaStream_t s, int64_t* launches,
                         const HaloPush& push);

// 3-D 7-point Jacobi (TMA-staged tiles) on planes [i0, i1) x rows [jl, jh) x cols [kl, kh) of an
// n0 x n1 x n2 fp32 array; needs n2 % 4 == 0 (else cudaErrorNotSupported).
// [src_lo, src_hi): the element range allocated behind src (the TMA map is limited to it).
cudaError_t jacobi3d(const float* src, float* dst, int64_t n0, int64_t n1, int64_t n2, int64_t i0, int64_t i1,
                     int64_t jl, int64_t jh, int64_t kl, int64_t kh, int64_t src_lo, int64_t src_hi, Track t,
                     cudaStream_t s, int64_t* launches);

// Deep-halo body fused (h sweeps per launch): register-streamed temporal blocking (one warp per 128-column strip marching
// down the rows, all h levels advanced per input row); 2 <= h <= 8.
cudaError_t jacobi2d_deep_stream(const float* src, float* dst, int64_t rows, int64_t cols, int64_t r0, int64_t r1,
                                 int64_t rlo, int64_t rhi, int64_t c0, int64_t c1, int h, int64_t src_lo,
                                 int64_t src_hi, Track t, cudaStream_t s, int64_t* launches);

// Deep-halo scratch frame: rows [lo, hi) of tmp get src's values outside the update box
// (rows outside [rlo, rhi) entirely, columns outside [c0, c1) of the others).
cudaError_t frame_copy(const float* src, float* tmp, int64_t cols, int64_t lo, int64_t hi, int64_t rlo, int64_t rhi,
                       int64_t c0, int64_t c1, cudaStream_t s, int64_t* launches);

// Test body: rows i in [r0, r1) with i % period == 0: out[i][:] = in[i][:] + 1.0f.
cudaError_t sparse_rows(const float* in, float* out, int64_t rows, int64_t cols, int64_t r0, int64_t r1,
                        int64_t period, Track t, cudaStream_t s, int64_t* launches);
// Test body: e in [e0, e1) with mask[e] != 0: out[e] = in[e] + 1.0f (warp-aggregated tracking).
cudaError_t masked_write(const float* in, const uint8_t* mask, float* out, int64_t e0, int64_t e1, Track t,
                         cudaStream_t s, int64_t* launches);

// k-means assignment + reductiontoarray over points [p0, p1): member[p] = argmin_c (fmaf chain),
// sums[member][j] += x*2^shift (int64), counts[member] += 1 into the partition's partials.
// err_flag (device int) is set to 1 if some x is not on the 2^-shift grid.
cudaError_t kmeans_assign(const float* x, const float* cen, int32_t* member, int64_t* sums, int64_t* counts,
                          int64_t p0, int64_t p1, int d, int kc, int shift, int* err_flag, cudaStream_t s,
                          int64_t* launches);
// Same loop with the distance cross term on the tcgen05 tensor cores and an exact fmaf re-check of
// the candidates (kmeans_tc.cu): d == 16, 1 <= kc <= 256, x 16-byte aligned.
int kmeans_tc_supported(const float* x, int d, int kc);
cudaError_t kmeans_assign_tc(const float* x, const float* cen, int32_t* member, int64_t* sums, int64_t* counts,
                             int64_t p0, int64_t p1, int kc, int shift, int* err_flag, cudaStream_t s, int sms);
// k-means update over clusters [c0, c1); tracked writes of centroids, sums, counts.
cudaError_t kmeans_update(int64_t* sums, int64_t* counts, float* cen, int64_t c0, int64_t c1, int d, int shift,
                          Track t_sums, Track t_counts, Track t_cen, cudaStream_t s, int64_t* launches);

// bf16 x bf16 -> fp32 GEMM of rows [m0, m1) of C = A.B (A [M][K], B [K][N], C [M][N], row-major),
// tcgen05.mma with TMEM accumulators and TMA operand staging.
// a_lo: first element of A's allocation (the A tensor map starts at its first whole row).
cudaError_t gemm_bf16(const uint16_t* A, const uint16_t* B, float* C, int64_t M, int64_t N, int64_t K,
                      int64_t m0, int64_t m1, int64_t a_lo, cudaStream_t s, int64_t* launches);

// Irregular-write body (L137): dst[idx[i]] = src[i] for i in [i0, i1); writes whose index is outside
// [wlo, whi) append {index, value bits} to recs (slot from *count, warp-aggregated).
cudaError_t scatter_body(const float* src, const int32_t* idx, float* dst, int64_t i0, int64_t i1, int64_t wlo,
                         int64_t whi, uint64_t* recs, int64_t* count, cudaStream_t s, int64_t* launches);
// Completes buffered writes in the owners' replicas: record (e, v) goes to dsts.p[h] where h is
// the window [bounds[h], his[h]) holding e (nb windows, ascending). count = device counter. A record
// no window holds is dropped and sets *bad.
cudaError_t apply_misses(const uint64_t* recs, const int64_t* count, int64_t cap, const PtrList& dsts,
                         const int64_t* bounds_dev, const int64_t* his_dev, int nb, int64_t* total, int* bad,
                         int64_t extent, cudaStream_t s, int64_t* launches);

// ---- coherence: compaction of dirty runs, scatter into peer replicas -------------------------
constexpr int kTileWords = 2048;   // bitmap words per compaction tile (65536 elements)

// Pass 1: per-tile counts {run starts, run ends, elements} of tiles holding a dirty chunk
// (chunks with a clear L2 bit are skipped without reading L1); also records each tile's first
// and last word (neighbours for pass 3, which clears L1 as it goes).
cudaError_t compact_count(const uint32_t* l1, const uint32_t* l2, int64_t nwords, int chunk_words_log2,
                          int64_t ntiles, int64_t* tile_counts, uint32_t* tile_edges, cudaStream_t s,
                          int64_t* launches);
// Pass 2 (one block): exclusive scan of the tile counts; totals[0..3] = {n_runs, n_elems,
// dirty_chunks, n_run_ends}; clears the L2 bits. (The packed header is totals[0..1].)
cudaError_t compact_scan(const int64_t* tile_counts, int64_t ntiles, int64_t* tile_offs, int64_t* totals,
                         uint32_t* l2, int64_t nl2words, cudaStream_t s, int64_t* launches);
// Pass 3: run starts/ends and payload into the canonical packed buffer; clears L1 words.
// values holds elements [0, extent) (global indices). push.n > 0:
// every dirty element is also stored at its global index into each replica of push (the other
// partitions' replicas, local or IPC-mapped peers): compaction and propagation in one pass.
cudaError_t compact_write(uint32_t* l1, int64_t nwords, int64_t extent, int64_t ntiles, const int64_t* tile_counts,
                          const int64_t* tile_offs, const uint32_t* tile_edges, const void* values,
                          int esize, uint8_t* packed, int64_t n_runs, const PtrList& push, cudaStream_t s,
                          int64_t* launches, int keep_packed = 1);
// Scatter the runs of a canonical packed buffer into ndst replicas at the same global indices.
// scratch: >= 2 * kScatterBlocks int64.
constexpr int kScatterBlocks = 592;  // 4 x 148 SMs (64 registers x 256 threads: 4 resident per SM)
cudaError_t scatter_packed(const uint8_t* packed, int64_t n_runs, const PtrList& dsts, int esize,
                           int64_t* scratch, cudaStream_t s, int64_t* launches);

// The paper's chunk protocol (L133-135): every dirty chunk's elements with a set L1 bit are copied
// from `values` into each destination replica; clears those L1 words.
cudaError_t chunk_merge(uint32_t* l1, const uint32_t* l2, int64_t nwords, int chunk_words_log2, const void* values,
                        int esize, const PtrList& dsts, cudaStream_t s, int64_t* launches);

// Batched device copies (data-loader pulls of one phase; src may be a peer's replica mapped
// through IPC, read over NVLink): up to kMaxCopies ranges in one launch.
constexpr int kMaxCopies = 32;
struct CopyList {
    void* dst[kMaxCopies];
    const void* src[kMaxCopies];
    int64_t bytes[kMaxCopies];
    int n;
};
cudaError_t copy_batch(const CopyList& c, cudaStream_t s, int64_t* launches);

// ---- reductions (reductiontoarray merge, L112) -------------------------------------------------
// acc[i] += srcs.p[j][i] for every j, then dsts.p[j][i] += acc[i] for every j (int64 elements).
cudaError_t reduce_sum_i64(int64_t* acc, const PtrList& srcs, int64_t n, cudaStream_t s, int64_t* launches);
cudaError_t apply_add_i64(const PtrList& dsts, const int64_t* acc, int64_t n, cudaStream_t s, int64_t* launches);

// Cross-process device barrier (p2p.cu): peer_sigs.p[q] = rank q's sig array (mapped via IPC).
cudaError_t device_barrier(const PtrList& peer_sigs, uint64_t* my_sig, int rank, int W, uint64_t epoch,
                           cudaStream_t s, int64_t* launches);

// Device-side bitwise AND test of two bitmaps (debug_checks): *flag |= any(a & b).
cudaError_t bitmap_overlap(const uint32_t* a, const uint32_t* b, int64_t nwords, int* flag, cudaStream_t s,
                           int64_t* launches);

}  // namespace k
}  // namespace accmg
