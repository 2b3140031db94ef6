// Internal definitions of libuniconn_b200 (not part of the C-ABI).
#pragma once

#include <cuda_runtime.h>
#include <nccl.h>

#include <cstdint>
#include <algorithm>
#include <cstdio>
#include <string>
#include <vector>

#include "uniconn.h"

namespace uc {

// ----------------------------------------------------------------------------- errors
void set_error(const std::string& msg);
int fail(int status, const char* fmt, ...);

#define UC_CUDA(call)                                                                        \
  do {                                                                                       \
    cudaError_t uc_e_ = (call);                                                              \
    if (uc_e_ != cudaSuccess)                                                                \
      return ::uc::fail(UC_ERR_CUDA, "%s failed at %s:%d: %s", #call, __FILE__, __LINE__,     \
                        cudaGetErrorString(uc_e_));                                          \
  } while (0)

#define UC_NCCL(call)                                                                        \
  do {                                                                                       \
    ncclResult_t uc_n_ = (call);                                                             \
    if (uc_n_ != ncclSuccess)                                                                \
      return ::uc::fail(UC_ERR_NCCL, "%s failed at %s:%d: %s", #call, __FILE__, __LINE__,     \
                        ncclGetErrorString(uc_n_));                                          \
  } while (0)

#define UC_TRY(call)                                                                         \
  do {                                                                                       \
    int uc_s_ = (call);                                                                      \
    if (uc_s_ != UC_OK) return uc_s_;                                                        \
  } while (0)

// ----------------------------------------------------------------------------- device-side shared structs
// Everything a device-mode Jacobi iteration needs, passed by value to the kernel.
struct JacobiParams {
  float* slab[2];          // local ping-pong slabs, (n+2) x nx each
  float* top_slab[2];      // top neighbour's slabs (nullptr when none)
  float* bot_slab[2];      // bottom neighbour's slabs
  uint64_t* my_flags;      // local: [0, S) from_top[s], [S, 2S) from_bottom[s] (stride kFlagStride)
  uint64_t* top_flags;     // top neighbour's flag array (we set its from_bottom[s])
  uint64_t* bot_flags;     // bottom neighbour's flag array (we set its from_top[s])
  // variant 4 (two iterations per launch): the A_{k+1} boundary rows travel through a second,
  // small symmetric buffer per rank: rows [2][nx] (0 = from top, 1 = from bottom) and per-strip
  // flags [2][flag_half] (from_top[s], from_bottom[s]; value k+1 = "A_{k+1} row present")
  float* h1_rows;          // local
  uint64_t* h1_flags;      // local
  float* top_h1_rows;      // top neighbour's (we write its "from bottom" row)
  uint64_t* top_h1_flags;
  float* bot_h1_rows;      // bottom neighbour's (we write its "from top" row)
  uint64_t* bot_h1_flags;
  double* norm_slot[UC_MAX_RANKS];     // rank q's norm slots: [2][P] doubles
  uint64_t* norm_flag[UC_MAX_RANKS];   // rank q's norm flags: [2][P] u64 (stride kFlagStride)
  unsigned long long* k_dev;           // local [k, norm round m, slab parity offset, -]
  unsigned long long* launch_hist;     // local [16]: completed launches by iterations per launch
  unsigned int* done;                  // local block ticket
  unsigned int* work;                  // local dynamic tile counter (variant 2)
  unsigned int* nbar;                  // local [count, generation] norm grid barrier (variant 3)
  uint64_t* blk_done;                  // local [grid] last iteration each block completed (variant 3)
  int tile_rows;                       // variant 2: rows per work item
  int strip4;                          // variant 5: owned float4 columns per strip (ghost-lane layout)
  int chunk_shrink;                    // variant 5: rows taken off the first/last row chunk
  int ghosts;                          // variant 5: ghost lanes per warp side (1: T <= 4, 2: T <= 8)
  int deep_halo;                       // variant 5, host mode: T halo rows per side with a neighbour
  int part;                            // variant 5: 0 whole launch, 1 edge chunks, 2 other chunks
  int partial_base;                    // index of this launch's first block partial
  unsigned put_delay_ns;               // test/measurement knob (UC_INJECT_PUT_DELAY_NS): each boundary
                                       // round's flag is released this much later (NVLink-like latency)
  // variant 5, device mode, norm-free launches: the balanced work table (nullptr: the static
  // chunking).  bal_tab[b] = {strip, chunk, first row, last row} of block b.  Launches of depth
  // bal_T time each block's march; their last block folds the times into the rates and re-cuts
  // every strip's rows in proportion to its blocks' rates
  int4* bal_tab;
  const int* bal_inv;                  // [strips * chunks]: block serving (strip s, chunk q) at s * chunks + q
  unsigned long long* bal_ns;          // [grid]: block b's march time in the last launch of depth bal_T
  float* bal_rate;                     // [grid]: block b's smoothed rate, rows per ns
  int bal_T;
  int bal_levels;                      // the solver's T (minimum chunk sizes)
  int gpu_scope;                       // 1: top and bottom live on this GPU (same process): halo
                                       // flags at .gpu scope instead of .sys
  double* partials;                    // local [grid] per-block partial sums
  double* rank_sum;                    // local: this rank's sum of squares (host-mode allreduce in place)
  double* norm_hist;                   // local: norms by round m (ring of norm_cap)
  unsigned int* err;                   // local error word (bit 0 = timeout)
  unsigned long long timeout_ns;
  int nx, n;               // columns, owned rows
  int nx4;                 // nx / 4
  int strips, chunks;      // grid = strips * chunks blocks
  int flag_half;           // from_bottom flags start at index flag_half (= max strips)
  int variant;             // 0: register y-march (LDG.128), 1: TMA-staged y-march (smem ring)
  int consumers;           // variant 1: compute threads per block (a producer warp comes on top)
  int stages;              // variant 1: ring depth (rows)
  int has_top, has_bot;
  int device_mode;         // 1: fused waits + puts + in-kernel cross-rank norm
  int norm_every;          // <= 0: never
  int norm_cap;
  int rank, size;
};

constexpr int kFlagStride = 16;  // u64 per flag = 128 bytes, one flag per L2 line
// Defaults from the round-1 sweeps at 16384^2 (profiles/r1_sweep.txt, r1_two_step_sweep.txt,
// r1_multi_step_sweep.txt): the TMA-staged march with a 3-row ring reaches 6.36 TB/s vs 6.07 for
// the register march (deeper rings lose); the two-iteration kernel (variant 4, 3 blocks/SM,
// 4-row ring) moves the same 8 B/point per launch at 6.4 TB/s for two iterations; the T-level
// ghost-lane kernel (variant 5, T = 4, 2 blocks/SM, 8-row ring) does four iterations per launch
// at 0.40 ms, so it is the default.
constexpr int kDefaultVariant = 5;
constexpr int kDefaultStages = 3;
constexpr int kDefaultStagesTwoStep = 4;
constexpr int kDefaultStagesMulti = 9;  // a multiple of the grouped march's kGroup (9)
constexpr int kDefaultTileRows = 64;

// Launch wrappers implemented in kernels.cu
int launch_jacobi_iteration(const JacobiParams& p, int grid, int block, cudaStream_t s);
int launch_jacobi_two_step(const JacobiParams& p, int grid, int block, cudaStream_t s);
int launch_jacobi_t(const JacobiParams& p, int grid, int block, int T, cudaStream_t s);
// host-overlap split launch: sum the block partials of both parts (norm launches), advance k by T
int launch_overlap_finish(const JacobiParams& p, int T, int nparts, cudaStream_t s);
// uc_jacobi_solve: the WHILE body's last kernel -- reads the period's norm, sets the condition
int launch_solve_check(const double* norm_hist, int norm_cap, const unsigned long long* k_dev, double tol,
                       unsigned long long kmax, cudaGraphConditionalHandle h, double* last, cudaStream_t s);
int preload_multistep();                                             // multistep.cu
// the deepest instance of a ghost layout (G = 1: T = 4; G = 2: T = 8) bounds the geometry of all T
int multistep_occupancy(int block, size_t smem, int ghosts, int* blocks_per_sm);
size_t multistep_smem_bytes(int consumers, int stages, int ghosts);  // the ring carries 4G halo floats per side
int launch_jacobi_t_g2(const JacobiParams& p, int grid, int block, int T, size_t smem, cudaStream_t s);  // multistep_g2.cu
int preload_multistep_g2();
int launch_jacobi_t_g2b(const JacobiParams& p, int grid, int block, int T, size_t smem, cudaStream_t s);  // multistep_g2b.cu
int preload_multistep_g2b();
int launch_jacobi_t_g2c(const JacobiParams& p, int grid, int block, size_t smem, cudaStream_t s);  // multistep_g2c.cu
int preload_multistep_g2c();
int multistep_occupancy_g2(int block, size_t smem, int* blocks_per_sm);
int multistep_max_consumers(int ghosts);
int multistep_stage_group();  // variant 5 ring stages: a multiple of this (grouped march)  // consumer threads per block the launch bounds allow
int launch_jacobi_persistent(const JacobiParams& p, int grid, int block, int iters, cudaStream_t s);
// Stream-ordered device -> host copy of n doubles on the coordinator's stream that never blocks
// the calling thread: into page-locked memory directly; into pageable memory into `stage`
// (page-locked, >= n doubles, owned by the caller) and from there into `host` at the next
// uc_coord_sync / uc_coord_destroy (the outputs' contract: valid after uc_coord_sync).  A plain
// pageable cudaMemcpyAsync returns only after the stream's earlier work, and with several ranks
// in one process that wait can stall a peer's launch behind a kernel waiting for that peer; a
// stream host function instead serialises on the driver's callback thread across streams.
// Inside a stream capture: a plain cudaMemcpyAsync.
int enqueue_d2h_f64(uc_coord* k, double* host, const double* dev, double* stage, size_t n);
int launch_norm_finish(double* rank_sum, double* norm_hist, int norm_cap, unsigned long long* k_dev,
                       int norm_every, cudaStream_t s);
int launch_init_field(float* slab0, float* slab1, int nx, int n, int ny, int row0, int ring,
                      int has_top, int has_bot, uint64_t seed, int zero_init, const float* colL,
                      const float* toprow, cudaStream_t s);
int launch_put_signal(const void* src, void* dst, size_t bytes, uint64_t* sig, uint64_t val,
                      unsigned int* counter, cudaStream_t s);
int launch_signal_wait(const uint64_t* sig, uint64_t val, unsigned long long timeout_ns, unsigned int* err,
                       cudaStream_t s);
int launch_allreduce_oneshot(const void* send, void* recv, size_t count, int dtype, int op, int root, int rank,
                             int size, void* const* peer_slots, uint64_t* const* peer_flags, const uint64_t* my_flags,
                             const void* my_slots, uint64_t epoch, size_t slot_bytes,
                             unsigned long long timeout_ns, unsigned int* err, cudaStream_t s);
// device-mode one-shot AllReduce (root < 0) / Reduce (to root) over the coordinator's slots
int oneshot_reduce(uc_coord* k, const void* send, void* recv, size_t count, uc_dtype dt, uc_redop op, int root);
int jacobi_occupancy(int variant, int block, size_t smem, int* blocks_per_sm);
struct P2PLaunch {
  const void* src;
  void *dst_peer, *dst_top, *dst_bot;
  uint64_t *sig_peer, *sig_top, *sig_bot, *sig_mine;
  unsigned int* bar;
  size_t bytes;
  uint64_t base;
  int iters, window, pattern, role, blocks;
  unsigned long long timeout_ns;
  unsigned int* err;
};
int launch_p2p_bench(const P2PLaunch& L, cudaStream_t s);
int launch_partial_ack(uint64_t* my_flags, uint64_t* top_flags, uint64_t* bot_flags, int strips, int flag_half,
                       const unsigned long long* k_dev, unsigned long long timeout_ns, unsigned int* err,
                       cudaStream_t s);
int launch_wait_halo(const uint64_t* my_flags, int strips, int flag_half, int has_top, int has_bot, uint64_t k,
                     unsigned long long timeout_ns, unsigned int* err, cudaStream_t s);
size_t staged_smem_bytes(int consumers, int stages);
int preload_kernels();
int preload_cg_kernels();
int ensure_nccl(uc_coord* k);
const void* builtin_kernel(const char* name);

}  // namespace uc

// ----------------------------------------------------------------------------- opaque handles
struct uc_env {
  int rank = 0, size = 1, device = 0;
  uc_allgather_fn ag = nullptr;
  void* ag_ctx = nullptr;
  int live_comms = 0;
  int allgather(const void* send, void* recv, size_t bytes);
};

struct PeerRecord {
  uint64_t host_hash;
  int32_t pid;
  int32_t device;
  int32_t top, bottom;
  int32_t rank;
  int32_t pad;
};

struct uc_comm {
  uc_env* env = nullptr;
  int rank = 0, size = 1, top = -1, bottom = -1;
  int topology = UC_TOPO_NONE;
  std::vector<PeerRecord> peers;
  int* dev_view = nullptr;  // {rank, size, top, bottom}
  int live_objects = 0;
  bool same_process(int r) const;
};

struct uc_mem {
  uc_comm* comm = nullptr;
  size_t bytes = 0;
  void* local = nullptr;
  std::vector<void*> ptrs;      // per rank
  std::vector<bool> ipc_opened; // per rank: close with cudaIpcCloseMemHandle
};

struct GraphCache;

struct uc_coord {
  uc_comm* comm = nullptr;
  uc_mode mode = UC_MODE_HOST;
  cudaStream_t stream = nullptr;
  ncclComm_t nccl = nullptr;
  int in_group = 0;
  unsigned long long timeout_ns = 10ull * 1000 * 1000 * 1000;
  unsigned int* err = nullptr;         // device error word
  unsigned int* put_counter = nullptr; // device counter for multi-block put_signal
  uc_mem* ar_scratch = nullptr;        // device-mode allreduce slots [2][P][slot_bytes] + flags
  size_t ar_slot_bytes = 32768;
  uint64_t ar_epoch = 0;
  uc_mem* coll_flags = nullptr;        // device/partial: [ready P][done P] flags of the collectives
  uint64_t coll_epoch = 0;
  float* nccl_scratch = nullptr;       // host-mode barrier operand
  uint64_t p2p_epoch[3][UC_MAX_RANKS] = {};  // signal base of the next uc_p2p_bench call, per (pattern, peer)
  unsigned int* p2p_bar = nullptr;     // grid barrier [count, gen] of the p2p kernel
  int put_path = 0, wait_path = 0;     // uc_coord_set_p2p_path: SM / copy engine, spin kernel / stream wait
  cudaStream_t side = nullptr;         // host-overlap path: NCCL halo exchange beside the interior
  cudaEvent_t ev_fork = nullptr, ev_join = nullptr;
  struct PendingCopy {
    double* dst;
    const double* src;
    size_t n;
  };
  std::vector<PendingCopy> pending;    // staged pageable outputs, copied at uc_coord_sync
  std::vector<GraphCache*> caches;     // solvers' graph caches holding graphs built on this coordinator
};

// A captured run.  The graph bakes in its coordinator's stream, error word, spin timeout and (host /
// partial mode) NCCL communicator, so the coordinator and its timeout are part of the key and a
// coordinator's graphs die with it (GraphCache::forget from uc_coord_destroy).
struct JacobiGraph {
  int iters = 0, norm_every = 0, parity = 0, flip = 0, mode = -1;
  cudaStream_t stream = nullptr;
  const uc_coord* coord = nullptr;
  unsigned long long timeout_ns = 0;
  cudaGraphExec_t exec = nullptr;
};

// The graphs one solver (Jacobi or CG) built, and the coordinators that know about this cache.
struct GraphCache {
  std::vector<JacobiGraph> graphs;
  std::vector<uc_coord*> coords;
  void add(uc_coord* k, const JacobiGraph& g);  // registers the cache with k
  void clear();                                 // destroy every graph (geometry change)
  void forget(uc_coord* k);                     // destroy k's graphs and unregister (k is being destroyed)
  void release();                               // solver destroyed: clear + unregister
};

struct uc_jacobi {
  uc_comm* comm = nullptr;
  int nx = 0, n = 0, ny = 0, row0 = 0;
  int ring = 0;
  int64_t k = 0;                 // host mirror of the device iteration counter k_dev[0]
  int64_t m = 0;                 // host mirror of the device norm-round counter k_dev[1]
  uc_mem* slabs = nullptr;       // symmetric: 2 * (n+2) * nx floats
  uc_mem* ctrl = nullptr;        // symmetric: flags + norm slots
  uc_mem* h1 = nullptr;          // symmetric: A_{k+1} boundary rows + flags (variant 4)
  int flip = 0;                  // host mirror of k_dev[2]: A_k lives in slab (k + flip) & 1
  int levels = 1;                // variant 5: iterations per launch T
  int strip4 = 0;                // variant 5: owned float4 columns per strip
  int chunk_shrink = 0;          // variant 5: rows taken off the first/last row chunk
  int ghosts = 1;                // variant 5: ghost lanes per warp side (2 when T > 4)
  size_t slab_elems = 0;         // (n+2) * nx: one slab view (halo rows included)
  size_t slab_stride = 0;        // (n + 2 kHaloRows) * nx: one slab in the allocation
  size_t slab_off = 0;           // (kHaloRows - 1) * nx: view row 0 within its slab
  int host_deep = 0;             // host mode: T halo rows exchanged once per T-iteration launch
  int host_overlap = 0;          // host mode: edge chunks -> NCCL on a side stream || other chunks
  int strips = 0;               // current column strips (launch geometry)
  int max_strips = 0;           // flag capacity per side = ceil(nx/4 / 32)
  // local device state
  unsigned long long* k_dev = nullptr;
  unsigned long long* launch_hist = nullptr;  // [16] completed launches by iterations per launch
  unsigned int* done = nullptr;
  double* partials = nullptr;
  uint64_t* blk_done = nullptr;  // [partials_cap] per-block completed iteration (variant 3)
  double* rank_sum = nullptr;
  double* norm_hist = nullptr;
  double* norm_stage = nullptr;  // page-locked mirror of norm_hist for pageable norm outputs
  int norm_cap = 4096;
  cudaStream_t aux = nullptr;    // private non-blocking stream (init, synchronous copies)
  int variant = uc::kDefaultVariant, consumers = 0, stages = 0, tile_rows = 0;
  int last_mode = -1;            // mode of the coordinator that ran the previous iterations
  int block = 0, blocks_per_sm = 0, grid = 0, chunks = 0;
  int partials_cap = 0;
  GraphCache graphs;
  // balanced work table (variant 5, device mode, norm-free launches): blocks are
  // placed on SMs the same way every launch and SMs differ in speed (up to ~1.3x, measured); the
  // table re-cuts the strips' rows in proportion to measured per-block rates.  Off by default:
  // it equalises the blocks' finish times, but the fast SMs slow down when given more rows
  // (the rates are shares of a common limit), so the launch gains ~2 % and the step nothing
  int balance = 0;                         // uc_jacobi_set_balance
  int bal_ok = 0;                          // the device table holds a valid partition
  int bal_cap = 0;                         // capacity of the arrays below (blocks)
  int4* bal_tab = nullptr;                 // device [cap]: {strip, chunk, first row, last row}
  int* bal_inv = nullptr;                  // device [cap]: (strip, chunk) -> block
  unsigned long long* bal_ns = nullptr;    // device [cap]: march ns of the last timed launch
  float* bal_rate = nullptr;               // device [cap]: smoothed rows per ns per block
  int4* bal_tab_h = nullptr;               // pinned staging of a table upload
  int* bal_inv_h = nullptr;                // pinned staging of an inverse upload
  float* bal_rate_h = nullptr;             // pinned readback of bal_rate
  cudaEvent_t bal_ev = nullptr;            // after the readback
  int bal_pending = 0;                     // a readback is in flight
  int bal_T = 0;                           // the depth whose launches are timed
  int bal_assigned = 0;                    // the host has dealt blocks to strips by measured rates
  std::vector<int> bal_strip;              // block -> strip of the table on the device
};

// Partition each strip's n rows among its `chunks` blocks in proportion to the blocks' rates
// (uc_balance_plan in the C-ABI; pure host logic).  Returns false when the minimum sizes do not fit.
bool balance_plan(int strips, int chunks, int n, int shrink, int levels, const double* rate, int4* tab,
                  const double* strip_cols = nullptr);
