// runtime.cpp -- Environment, Communicator, Memory and Coordinator of libuniconn_b200
// (§IV), plus the P2P (Post/Acknowledge) and AllReduce
// primitives.  Host code only; kernels live in kernels.cu.
#include <cuda.h>
#include <unistd.h>

#include <cstdarg>
#include <cstring>
#include <fstream>
#include <functional>
#include <string>

#include "uc_internal.h"

namespace uc {

static thread_local std::string g_last_error;

void set_error(const std::string& msg) { g_last_error = msg; }

int fail(int status, const char* fmt, ...) {
  char buf[1024];
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(buf, sizeof buf, fmt, ap);
  va_end(ap);
  g_last_error = std::string(uc_status_string(status)) + ": " + buf;
  return status;
}

static void flush_pending(uc_coord* k);

int enqueue_d2h_f64(uc_coord* k, double* host, const double* dev, double* stage, size_t n) {
  if (!host || n == 0) return UC_OK;
  cudaStreamCaptureStatus cs = cudaStreamCaptureStatusNone;
  UC_CUDA(cudaStreamIsCapturing(k->stream, &cs));
  cudaPointerAttributes a{};
  const bool pinned = cudaPointerGetAttributes(&a, host) == cudaSuccess && a.type != cudaMemoryTypeUnregistered;
  cudaGetLastError();  // clear a failed query
  if (pinned || !stage || cs != cudaStreamCaptureStatusNone) {
    UC_CUDA(cudaMemcpyAsync(host, dev, n * sizeof(double), cudaMemcpyDeviceToHost, k->stream));
    return UC_OK;
  }
  // a stage slot still pending (more than the history's worth of outputs enqueued since the
  // last uc_coord_sync) is completed first, so the earlier output never receives a later value
  for (const auto& c : k->pending)
    if (c.src < stage + n && stage < c.src + c.n) {
      UC_CUDA(cudaStreamSynchronize(k->stream));
      flush_pending(k);
      break;
    }
  UC_CUDA(cudaMemcpyAsync(stage, dev, n * sizeof(double), cudaMemcpyDeviceToHost, k->stream));
  k->pending.push_back({host, stage, n});
  return UC_OK;
}

static void flush_pending(uc_coord* k) {
  for (const auto& c : k->pending) memcpy(c.dst, c.src, c.n * sizeof(double));
  k->pending.clear();
}

static uint64_t host_hash() {
  std::string id;
  char name[256] = {0};
  gethostname(name, sizeof name - 1);
  id = name;
  std::ifstream f("/proc/sys/kernel/random/boot_id");
  std::string boot;
  if (f) std::getline(f, boot);
  id += "|" + boot;
  return (uint64_t)std::hash<std::string>{}(id);
}

}  // namespace uc

using namespace uc;

void GraphCache::add(uc_coord* k, const JacobiGraph& g) {
  graphs.push_back(g);
  if (std::find(coords.begin(), coords.end(), k) == coords.end()) {
    coords.push_back(k);
    k->caches.push_back(this);
  }
}

void GraphCache::clear() {
  for (auto& g : graphs) cudaGraphExecDestroy(g.exec);
  graphs.clear();
}

void GraphCache::forget(uc_coord* k) {
  for (auto it = graphs.begin(); it != graphs.end();) {
    if (it->coord == k) {
      cudaGraphExecDestroy(it->exec);
      it = graphs.erase(it);
    } else {
      ++it;
    }
  }
  coords.erase(std::remove(coords.begin(), coords.end(), k), coords.end());
  k->caches.erase(std::remove(k->caches.begin(), k->caches.end(), this), k->caches.end());
}

void GraphCache::release() {
  clear();
  for (uc_coord* k : coords) k->caches.erase(std::remove(k->caches.begin(), k->caches.end(), this), k->caches.end());
  coords.clear();
}


int uc_env::allgather(const void* send, void* recv, size_t bytes) {
  if (size == 1) {
    memcpy(recv, send, bytes);
    return UC_OK;
  }
  if (!ag) return fail(UC_ERR_BOOTSTRAP, "world_size %d > 1 but no allgather callback", size);
  int rc = ag(send, recv, bytes, ag_ctx);
  if (rc != 0) return fail(UC_ERR_BOOTSTRAP, "allgather callback returned %d", rc);
  return UC_OK;
}

bool uc_comm::same_process(int r) const {
  const PeerRecord& me = peers[rank];
  return peers[r].host_hash == me.host_hash && peers[r].pid == me.pid;
}

extern "C" {

const char* uc_status_string(int s) {
  switch (s) {
    case UC_OK: return "UC_OK";
    case UC_ERR_ARG: return "UC_ERR_ARG";
    case UC_ERR_CUDA: return "UC_ERR_CUDA";
    case UC_ERR_NCCL: return "UC_ERR_NCCL";
    case UC_ERR_BOOTSTRAP: return "UC_ERR_BOOTSTRAP";
    case UC_ERR_TIMEOUT: return "UC_ERR_TIMEOUT";
    case UC_ERR_STATE: return "UC_ERR_STATE";
    case UC_ERR_UNSUPPORTED: return "UC_ERR_UNSUPPORTED";
    case UC_ERR_OOM: return "UC_ERR_OOM";
    default: return "UC_ERR_UNKNOWN";
  }
}

const char* uc_last_error(void) { return g_last_error.c_str(); }

int uc_version(void) { return 100; }

// ============================================================================ Environment
int uc_env_init(int world_rank, int world_size, int device, uc_allgather_fn ag, void* ag_ctx, uc_env** out) {
  if (!out) return fail(UC_ERR_ARG, "out is NULL");
  *out = nullptr;
  if (world_size < 1 || world_size > UC_MAX_RANKS)
    return fail(UC_ERR_ARG, "world_size %d not in [1, %d]", world_size, UC_MAX_RANKS);
  if (world_rank < 0 || world_rank >= world_size) return fail(UC_ERR_ARG, "world_rank %d out of range", world_rank);
  if (device != -1) {  // device == -1: bootstrap-only env (no GPU calls; CPU tests of the host logic)
    int ndev = 0;
    UC_CUDA(cudaGetDeviceCount(&ndev));
    if (device < 0 || device >= ndev) return fail(UC_ERR_ARG, "device %d not in [0, %d)", device, ndev);
    UC_CUDA(cudaSetDevice(device));
    UC_CUDA(cudaFree(nullptr));  // create the primary context now
    UC_TRY(preload_kernels());   // no lazy module loads once ranks spin on each other
    UC_TRY(preload_cg_kernels());
  }
  uc_env* e = new uc_env;
  e->rank = world_rank;
  e->size = world_size;
  e->device = device;
  e->ag = ag;
  e->ag_ctx = ag_ctx;
  *out = e;
  return UC_OK;
}

int uc_env_finalize(uc_env* env) {
  if (!env) return fail(UC_ERR_ARG, "env is NULL");
  if (env->live_comms) return fail(UC_ERR_STATE, "%d communicator(s) still alive", env->live_comms);
  delete env;
  return UC_OK;
}

int uc_env_info(const uc_env* env, int* rank, int* size, int* device) {
  if (!env) return fail(UC_ERR_ARG, "env is NULL");
  if (rank) *rank = env->rank;
  if (size) *size = env->size;
  if (device) *device = env->device;
  return UC_OK;
}

// ============================================================================ Communicator
int uc_comm_create(uc_env* env, int top, int bottom, uc_comm** out) {
  if (!env || !out) return fail(UC_ERR_ARG, "NULL argument");
  *out = nullptr;
  const int P = env->size, r = env->rank;
  if (top < -1 || top >= P || bottom < -1 || bottom >= P)
    return fail(UC_ERR_ARG, "neighbours (%d, %d) out of range for size %d", top, bottom, P);
  if (env->device >= 0) UC_CUDA(cudaSetDevice(env->device));
  PeerRecord me{};
  me.host_hash = host_hash();
  me.pid = (int32_t)getpid();
  me.device = env->device;
  me.top = top;
  me.bottom = bottom;
  me.rank = r;
  std::vector<PeerRecord> all(P);
  UC_TRY(env->allgather(&me, all.data(), sizeof(PeerRecord)));
  for (int q = 0; q < P; ++q) {
    if (all[q].rank != q) return fail(UC_ERR_BOOTSTRAP, "allgather slot %d holds rank %d", q, all[q].rank);
    if (all[q].top >= 0 && all[all[q].top].bottom != q)
      return fail(UC_ERR_ARG, "rank %d has top %d but rank %d's bottom is %d", q, all[q].top, all[q].top,
                  all[all[q].top].bottom);
    if (all[q].bottom >= 0 && all[all[q].bottom].top != q)
      return fail(UC_ERR_ARG, "rank %d has bottom %d but rank %d's top is %d", q, all[q].bottom, all[q].bottom,
                  all[all[q].bottom].top);
  }
  bool ring = true, chain = true;
  for (int q = 0; q < P; ++q) {
    const int rt = (q - 1 + P) % P, rb = (q + 1) % P;
    if (all[q].top != rt || all[q].bottom != rb) ring = false;
    const int ct = q == 0 ? -1 : q - 1, cb = q == P - 1 ? -1 : q + 1;
    if (all[q].top != ct || all[q].bottom != cb) chain = false;
  }
  uc_comm* c = new uc_comm;
  c->env = env;
  c->rank = r;
  c->size = P;
  c->top = top;
  c->bottom = bottom;
  c->topology = ring ? UC_TOPO_RING : chain ? UC_TOPO_CHAIN : UC_TOPO_NONE;
  c->peers = all;
  if (env->device >= 0) {
    int view[4] = {r, P, top, bottom};
    cudaError_t e = cudaMalloc(&c->dev_view, sizeof view);
    if (e == cudaSuccess) e = cudaMemcpy(c->dev_view, view, sizeof view, cudaMemcpyHostToDevice);
    if (e != cudaSuccess) {
      delete c;
      return fail(UC_ERR_CUDA, "device view: %s", cudaGetErrorString(e));
    }
  }
  env->live_comms++;
  *out = c;
  return UC_OK;
}

int uc_comm_destroy(uc_comm* c) {
  if (!c) return fail(UC_ERR_ARG, "comm is NULL");
  if (c->live_objects) return fail(UC_ERR_STATE, "%d object(s) still alive on this communicator", c->live_objects);
  if (c->env->device >= 0) {
    cudaSetDevice(c->env->device);
    cudaFree(c->dev_view);
  }
  c->env->live_comms--;
  delete c;
  return UC_OK;
}

int uc_comm_info(const uc_comm* c, int* rank, int* size, int* top, int* bottom, int* topology) {
  if (!c) return fail(UC_ERR_ARG, "comm is NULL");
  if (rank) *rank = c->rank;
  if (size) *size = c->size;
  if (top) *top = c->top;
  if (bottom) *bottom = c->bottom;
  if (topology) *topology = c->topology;
  return UC_OK;
}

int uc_comm_device_view(const uc_comm* c, const void** dev_ptr) {
  if (!c || !dev_ptr) return fail(UC_ERR_ARG, "NULL argument");
  if (c->env->device < 0) return fail(UC_ERR_STATE, "bootstrap-only environment has no device");
  *dev_ptr = c->dev_view;
  return UC_OK;
}

int uc_comm_barrier(uc_comm* c, void* stream) {
  if (!c) return fail(UC_ERR_ARG, "comm is NULL");
  if (c->env->device >= 0) {
    UC_CUDA(cudaSetDevice(c->env->device));
    UC_CUDA(cudaStreamSynchronize((cudaStream_t)stream));
  }
  std::vector<char> sink(c->size);
  char one = 1;
  return c->env->allgather(&one, sink.data(), 1);
}

// ============================================================================ Memory
struct IpcRecord {
  cudaIpcMemHandle_t handle;
  uint64_t raw;
  int32_t ok;
  int32_t pad;
};

int uc_mem_alloc_symmetric(uc_comm* c, size_t bytes, uc_mem** out) {
  if (!c || !out) return fail(UC_ERR_ARG, "NULL argument");
  *out = nullptr;
  if (bytes == 0) return fail(UC_ERR_ARG, "bytes == 0");
  if (c->env->device < 0) return fail(UC_ERR_STATE, "bootstrap-only environment has no device");
  UC_CUDA(cudaSetDevice(c->env->device));
  // agree on the size first (collective contract)
  std::vector<uint64_t> sizes(c->size);
  uint64_t b64 = bytes;
  UC_TRY(c->env->allgather(&b64, sizes.data(), sizeof b64));
  for (int q = 0; q < c->size; ++q)
    if (sizes[q] != b64) return fail(UC_ERR_ARG, "symmetric alloc size mismatch: rank %d asked %llu, rank %d %llu",
                                     c->rank, (unsigned long long)b64, q, (unsigned long long)sizes[q]);
  void* p = nullptr;
  cudaError_t e = cudaMalloc(&p, bytes);
  if (e != cudaSuccess) {
    cudaGetLastError();
    return fail(UC_ERR_OOM, "cudaMalloc(%zu): %s", bytes, cudaGetErrorString(e));
  }
  UC_CUDA(cudaMemset(p, 0, bytes));
  UC_CUDA(cudaStreamSynchronize(nullptr));
  IpcRecord rec{};
  rec.raw = (uint64_t)(uintptr_t)p;
  bool need_ipc = false;
  for (int q = 0; q < c->size; ++q)
    if (!c->same_process(q)) need_ipc = true;
  rec.ok = 1;
  if (need_ipc) {
    e = cudaIpcGetMemHandle(&rec.handle, p);
    if (e != cudaSuccess) {
      cudaGetLastError();
      rec.ok = 0;
    }
  }
  std::vector<IpcRecord> all(c->size);
  int rc = c->env->allgather(&rec, all.data(), sizeof rec);
  if (rc != UC_OK) {
    cudaFree(p);
    return rc;
  }
  uc_mem* m = new uc_mem;
  m->comm = c;
  m->bytes = bytes;
  m->local = p;
  m->ptrs.assign(c->size, nullptr);
  m->ipc_opened.assign(c->size, false);
  for (int q = 0; q < c->size; ++q) {
    if (q == c->rank) {
      m->ptrs[q] = p;
    } else if (c->same_process(q)) {
      m->ptrs[q] = (void*)(uintptr_t)all[q].raw;
      if (c->peers[q].device != c->env->device) {
        e = cudaDeviceEnablePeerAccess(c->peers[q].device, 0);
        if (e != cudaSuccess && e != cudaErrorPeerAccessAlreadyEnabled) {
          cudaGetLastError();
          m->ptrs[q] = nullptr;
        } else {
          cudaGetLastError();
        }
      }
    } else if (all[q].ok) {
      void* mp = nullptr;
      e = cudaIpcOpenMemHandle(&mp, all[q].handle, cudaIpcMemLazyEnablePeerAccess);
      if (e == cudaSuccess) {
        m->ptrs[q] = mp;
        m->ipc_opened[q] = true;
      } else {
        cudaGetLastError();
      }
    }
  }
  // every rank must be able to reach the peers the protocols use; report the first gap
  int unreachable = -1;
  for (int q = 0; q < c->size; ++q)
    if (!m->ptrs[q]) unreachable = q;
  c->live_objects++;
  *out = m;
  if (unreachable >= 0) {
    // not fatal for host-mode use; device-mode users check uc_mem_ptr
    set_error("uc_mem_alloc_symmetric: rank " + std::to_string(unreachable) + " not peer-addressable");
  }
  return UC_OK;
}

void* uc_mem_ptr(const uc_mem* m, int rank) {
  if (!m || rank < 0 || rank >= (int)m->ptrs.size()) return nullptr;
  return m->ptrs[rank];
}

size_t uc_mem_size(const uc_mem* m) { return m ? m->bytes : 0; }

int uc_mem_free_symmetric(uc_mem* m) {
  if (!m) return fail(UC_ERR_ARG, "mem is NULL");
  uc_comm* c = m->comm;
  UC_CUDA(cudaSetDevice(c->env->device));
  UC_CUDA(cudaStreamSynchronize(nullptr));
  UC_TRY(uc_comm_barrier(c, nullptr));  // nobody still writes into our buffer
  for (int q = 0; q < c->size; ++q)
    if (m->ipc_opened[q]) cudaIpcCloseMemHandle(m->ptrs[q]);
  UC_TRY(uc_comm_barrier(c, nullptr));  // nobody still maps our buffer
  cudaFree(m->local);
  c->live_objects--;
  delete m;
  return UC_OK;
}

}  // extern "C"

// NCCL communicator of a coordinator, created on first need (COLLECTIVE: every rank reaches
// it through the same collective call; the unique id travels over the bootstrap allgather).
int uc::ensure_nccl(uc_coord* k) {
  if (k->nccl) return UC_OK;
  uc_comm* c = k->comm;
  ncclUniqueId id{};
  if (c->rank == 0) UC_NCCL(ncclGetUniqueId(&id));
  std::vector<ncclUniqueId> ids(c->size);
  UC_TRY(c->env->allgather(&id, ids.data(), sizeof id));
  UC_NCCL(ncclCommInitRank(&k->nccl, c->size, ids[0], c->rank));
  return UC_OK;
}

extern "C" {

// ============================================================================ Coordinator
int uc_coord_create(uc_comm* c, uc_mode mode, void* stream, uc_coord** out) {
  if (!c || !out) return fail(UC_ERR_ARG, "NULL argument");
  *out = nullptr;
  if (mode != UC_MODE_HOST && mode != UC_MODE_DEVICE && mode != UC_MODE_PARTIAL)
    return fail(UC_ERR_ARG, "unknown mode %d", (int)mode);
  if (c->env->device < 0) return fail(UC_ERR_STATE, "bootstrap-only environment has no device");
  UC_CUDA(cudaSetDevice(c->env->device));
  uc_coord* k = new uc_coord;
  k->comm = c;
  k->mode = mode;
  k->stream = (cudaStream_t)stream;
  auto cleanup = [&](int rc) {
    if (k->err) cudaFree(k->err);
    if (k->put_counter) cudaFree(k->put_counter);
    if (k->nccl_scratch) cudaFree(k->nccl_scratch);
    if (k->nccl) ncclCommDestroy(k->nccl);
    delete k;
    return rc;
  };
  cudaError_t e = cudaMalloc(&k->err, sizeof(unsigned int));
  if (e == cudaSuccess) e = cudaMemset(k->err, 0, sizeof(unsigned int));
  // [0] put_signal block ticket, [1..2] p2p benchmark grid barrier (count, generation)
  if (e == cudaSuccess) e = cudaMalloc(&k->put_counter, 4 * sizeof(unsigned int));
  if (e == cudaSuccess) e = cudaMemset(k->put_counter, 0, 4 * sizeof(unsigned int));
  k->p2p_bar = k->put_counter + 1;
  if (e == cudaSuccess) e = cudaMalloc(&k->nccl_scratch, sizeof(float));
  if (e == cudaSuccess) e = cudaMemset(k->nccl_scratch, 0, sizeof(float));
  if (e == cudaSuccess) e = cudaStreamSynchronize(nullptr);
  if (e != cudaSuccess) return cleanup(fail(UC_ERR_CUDA, "coordinator state: %s", cudaGetErrorString(e)));
  // host mode: NCCL for everything; partial mode: NCCL for collectives, created at the
  // first collective, + peer memory for the in-kernel posts; device mode: peer memory only
  if (mode == UC_MODE_HOST) {
    int rc = ensure_nccl(k);
    if (rc != UC_OK) return cleanup(rc);
  }
  if (mode != UC_MODE_HOST) {
    const size_t P = (size_t)c->size;
    const size_t bytes = 2 * P * k->ar_slot_bytes + 2 * P * kFlagStride * sizeof(uint64_t);
    int rc = uc_mem_alloc_symmetric(c, bytes, &k->ar_scratch);
    if (rc != UC_OK) return cleanup(rc);
    for (int q = 0; q < c->size; ++q)
      if (!uc_mem_ptr(k->ar_scratch, q)) {
        uc_mem_free_symmetric(k->ar_scratch);
        return cleanup(fail(UC_ERR_UNSUPPORTED, "device mode needs every rank peer-addressable; rank %d is not", q));
      }
    rc = uc_mem_alloc_symmetric(c, 2 * P * kFlagStride * sizeof(uint64_t), &k->coll_flags);
    if (rc != UC_OK) {
      uc_mem_free_symmetric(k->ar_scratch);
      return cleanup(rc);
    }
  }
  c->live_objects++;
  *out = k;
  return UC_OK;
}

int uc_coord_destroy(uc_coord* k) {
  if (!k) return fail(UC_ERR_ARG, "coord is NULL");
  UC_CUDA(cudaSetDevice(k->comm->env->device));
  if (cudaStreamSynchronize(k->stream) == cudaSuccess) flush_pending(k);
  // solvers' graphs captured on this coordinator point at its error word / NCCL communicator:
  // they go with it (a later coordinator never replays them)
  while (!k->caches.empty()) k->caches.back()->forget(k);
  if (k->nccl) ncclCommDestroy(k->nccl);
  if (k->ar_scratch) UC_TRY(uc_mem_free_symmetric(k->ar_scratch));
  if (k->coll_flags) UC_TRY(uc_mem_free_symmetric(k->coll_flags));
  cudaFree(k->err);
  cudaFree(k->put_counter);
  cudaFree(k->nccl_scratch);
  if (k->side) cudaStreamDestroy(k->side);
  if (k->ev_fork) cudaEventDestroy(k->ev_fork);
  if (k->ev_join) cudaEventDestroy(k->ev_join);
  k->comm->live_objects--;
  delete k;
  return UC_OK;
}

int uc_coord_sync(uc_coord* k) {
  if (!k) return fail(UC_ERR_ARG, "coord is NULL");
  UC_CUDA(cudaSetDevice(k->comm->env->device));
  UC_CUDA(cudaStreamSynchronize(k->stream));
  flush_pending(k);
  unsigned int err = 0;
  UC_CUDA(cudaMemcpy(&err, k->err, sizeof err, cudaMemcpyDeviceToHost));
  if (err) {
    unsigned int zero = 0;
    UC_CUDA(cudaMemcpy(k->err, &zero, sizeof zero, cudaMemcpyHostToDevice));
    return fail(UC_ERR_TIMEOUT, "a device spin-wait exceeded %.3f s (error word 0x%x)", k->timeout_ns / 1e9, err);
  }
  if (k->nccl) {
    ncclResult_t ar = ncclSuccess;
    UC_NCCL(ncclCommGetAsyncError(k->nccl, &ar));
    if (ar != ncclSuccess) return fail(UC_ERR_NCCL, "NCCL async error: %s", ncclGetErrorString(ar));
  }
  return UC_OK;
}

int uc_coord_set_timeout(uc_coord* k, uint64_t timeout_ns) {
  if (!k || timeout_ns == 0) return fail(UC_ERR_ARG, "bad argument");
  k->timeout_ns = timeout_ns;
  return UC_OK;
}

typedef CUresult (*cuLaunchKernel_pfn)(CUfunction, unsigned, unsigned, unsigned, unsigned, unsigned, unsigned,
                                       unsigned, CUstream, void**, void**);

int uc_launch(uc_coord* k, const void* cu_function, unsigned gx, unsigned gy, unsigned gz, unsigned bx, unsigned by,
              unsigned bz, size_t smem_bytes, void** args) {
  if (!k || !cu_function) return fail(UC_ERR_ARG, "NULL argument");
  UC_CUDA(cudaSetDevice(k->comm->env->device));
  static cuLaunchKernel_pfn launch = nullptr;
  if (!launch) {
    void* fn = nullptr;
    cudaDriverEntryPointQueryResult q;
    UC_CUDA(cudaGetDriverEntryPoint("cuLaunchKernel", &fn, cudaEnableDefault, &q));
    if (q != cudaDriverEntryPointSuccess || !fn) return fail(UC_ERR_CUDA, "cuLaunchKernel entry point not found");
    launch = (cuLaunchKernel_pfn)fn;
  }
  CUresult r = launch((CUfunction)cu_function, gx, gy, gz, bx, by, bz, (unsigned)smem_bytes, (CUstream)k->stream,
                      args, nullptr);
  if (r != CUDA_SUCCESS) return fail(UC_ERR_CUDA, "cuLaunchKernel failed with CUresult %d", (int)r);
  return UC_OK;
}

int uc_builtin_kernel(const char* name, const void** cu_function) {
  if (!name || !cu_function) return fail(UC_ERR_ARG, "NULL argument");
  const void* sym = builtin_kernel(name);
  if (!sym) return fail(UC_ERR_ARG, "no builtin kernel named '%s'", name);
  cudaFunction_t f = nullptr;
  UC_CUDA(cudaGetFuncBySymbol(&f, sym));
  *cu_function = (const void*)f;
  return UC_OK;
}

int uc_group_start(uc_coord* k) {
  if (!k) return fail(UC_ERR_ARG, "coord is NULL");
  if (k->in_group) return fail(UC_ERR_STATE, "uc_group_start while a group is open");
  if (k->mode == UC_MODE_HOST) UC_NCCL(ncclGroupStart());
  k->in_group = 1;
  return UC_OK;
}

int uc_group_end(uc_coord* k) {
  if (!k) return fail(UC_ERR_ARG, "coord is NULL");
  if (!k->in_group) return fail(UC_ERR_STATE, "uc_group_end without uc_group_start");
  k->in_group = 0;
  if (k->mode == UC_MODE_HOST) {
    UC_CUDA(cudaSetDevice(k->comm->env->device));
    UC_NCCL(ncclGroupEnd());
  }
  return UC_OK;
}

// ============================================================================ P2P
int uc_put_signal(uc_coord* k, const void* src, uc_mem* dst, size_t dst_off, size_t bytes, uc_mem* sig,
                  size_t sig_idx, uint64_t sig_val, int peer) {
  if (!k || !src) return fail(UC_ERR_ARG, "NULL argument");
  uc_comm* c = k->comm;
  if (peer < 0 || peer >= c->size) return fail(UC_ERR_ARG, "peer %d out of range", peer);
  UC_CUDA(cudaSetDevice(c->env->device));
  if (k->mode == UC_MODE_HOST) {
    UC_NCCL(ncclSend(src, bytes, ncclUint8, peer, k->nccl, k->stream));
    return UC_OK;
  }
  if (!dst) return fail(UC_ERR_ARG, "dst is NULL in device mode");
  if (dst_off + bytes > dst->bytes) return fail(UC_ERR_ARG, "put of %zu bytes at %zu exceeds %zu", bytes, dst_off, dst->bytes);
  if (((uintptr_t)src | dst_off) & 15) return fail(UC_ERR_ARG, "src and dst_off must be 16-byte aligned");
  char* d = (char*)uc_mem_ptr(dst, peer);
  if (!d) return fail(UC_ERR_UNSUPPORTED, "rank %d is not peer-addressable", peer);
  uint64_t* s = nullptr;
  if (sig) {
    if ((sig_idx + 1) * sizeof(uint64_t) > sig->bytes) return fail(UC_ERR_ARG, "sig_idx %zu out of range", sig_idx);
    s = (uint64_t*)uc_mem_ptr(sig, peer);
    if (!s) return fail(UC_ERR_UNSUPPORTED, "rank %d signal not peer-addressable", peer);
    s += sig_idx;
  }
  if (k->put_path == UC_PUT_CE) {
    // copy engine over NVLink (a peer D2D copy), then the signal from a one-block kernel that
    // runs after the copy has completed (stream order)
    if (bytes) UC_CUDA(cudaMemcpyAsync(d + dst_off, src, bytes, cudaMemcpyDeviceToDevice, k->stream));
    return launch_put_signal(src, d + dst_off, 0, s, sig_val, k->put_counter, k->stream);
  }
  return launch_put_signal(src, d + dst_off, bytes, s, sig_val, k->put_counter, k->stream);
}

namespace {
typedef CUresult (*cuStreamWaitValue64_pfn)(CUstream, CUdeviceptr, cuuint64_t, unsigned int);
typedef CUresult (*cuDeviceGetAttribute_pfn)(int*, CUdevice_attribute, CUdevice);

// cuStreamWaitValue64(GEQ [| FLUSH]) through the driver entry point (no -lcuda link)
int stream_wait_ge(uc_coord* k, const uint64_t* sig, uint64_t val) {
  static cuStreamWaitValue64_pfn wait = nullptr;
  static cuDeviceGetAttribute_pfn attr = nullptr;
  if (!wait) {
    void* fn = nullptr;
    cudaDriverEntryPointQueryResult q;
    UC_CUDA(cudaGetDriverEntryPoint("cuStreamWaitValue64", &fn, cudaEnableDefault, &q));
    if (q != cudaDriverEntryPointSuccess || !fn) return fail(UC_ERR_UNSUPPORTED, "cuStreamWaitValue64 not available");
    wait = (cuStreamWaitValue64_pfn)fn;
    UC_CUDA(cudaGetDriverEntryPoint("cuDeviceGetAttribute", &fn, cudaEnableDefault, &q));
    if (q == cudaDriverEntryPointSuccess) attr = (cuDeviceGetAttribute_pfn)fn;
  }
  unsigned flags = CU_STREAM_WAIT_VALUE_GEQ;
  int ok64 = 1, flush = 0;
  if (attr) {
    attr(&ok64, CU_DEVICE_ATTRIBUTE_CAN_USE_64_BIT_STREAM_MEM_OPS, (CUdevice)k->comm->env->device);
    attr(&flush, CU_DEVICE_ATTRIBUTE_CAN_FLUSH_REMOTE_WRITES, (CUdevice)k->comm->env->device);
  }
  if (!ok64) return fail(UC_ERR_UNSUPPORTED, "device lacks 64-bit stream memory operations");
  if (flush) flags |= CU_STREAM_WAIT_VALUE_FLUSH;
  const CUresult r = wait((CUstream)k->stream, (CUdeviceptr)(uintptr_t)sig, (cuuint64_t)val, flags);
  if (r == CUDA_ERROR_NOT_SUPPORTED) return fail(UC_ERR_UNSUPPORTED, "cuStreamWaitValue64 not supported here");
  if (r != CUDA_SUCCESS) return fail(UC_ERR_CUDA, "cuStreamWaitValue64 failed with CUresult %d", (int)r);
  return UC_OK;
}
}  // namespace

int uc_coord_set_p2p_path(uc_coord* k, int put_path, int wait_path) {
  if (!k) return fail(UC_ERR_ARG, "coord is NULL");
  if (put_path != UC_PUT_SM && put_path != UC_PUT_CE) return fail(UC_ERR_ARG, "put_path %d", put_path);
  if (wait_path != UC_WAIT_KERNEL && wait_path != UC_WAIT_STREAM) return fail(UC_ERR_ARG, "wait_path %d", wait_path);
  k->put_path = put_path;
  k->wait_path = wait_path;
  return UC_OK;
}

int uc_signal_wait(uc_coord* k, uc_mem* dst, size_t dst_off, size_t bytes, uc_mem* sig, size_t sig_idx,
                   uint64_t sig_val, int peer) {
  if (!k) return fail(UC_ERR_ARG, "coord is NULL");
  uc_comm* c = k->comm;
  UC_CUDA(cudaSetDevice(c->env->device));
  if (k->mode == UC_MODE_HOST) {
    if (!dst) return fail(UC_ERR_ARG, "dst is NULL");
    if (peer < 0 || peer >= c->size) return fail(UC_ERR_ARG, "peer %d out of range", peer);
    if (dst_off + bytes > dst->bytes) return fail(UC_ERR_ARG, "recv exceeds buffer");
    UC_NCCL(ncclRecv((char*)dst->local + dst_off, bytes, ncclUint8, peer, k->nccl, k->stream));
    return UC_OK;
  }
  if (!sig) return fail(UC_ERR_ARG, "sig is NULL in device mode");
  if ((sig_idx + 1) * sizeof(uint64_t) > sig->bytes) return fail(UC_ERR_ARG, "sig_idx %zu out of range", sig_idx);
  if (k->wait_path == UC_WAIT_STREAM) return stream_wait_ge(k, (const uint64_t*)sig->local + sig_idx, sig_val);
  return launch_signal_wait((const uint64_t*)sig->local + sig_idx, sig_val, k->timeout_ns, k->err, k->stream);
}

// ============================================================================ AllReduce
int uc_p2p_bench(uc_coord* k, int pattern, uc_mem* buf, uc_mem* sig, size_t bytes, int iters, int window, int peer,
                 int role, int blocks) {
  if (!k || !buf || !sig) return fail(UC_ERR_ARG, "NULL argument");
  if (k->mode == UC_MODE_HOST) return fail(UC_ERR_UNSUPPORTED, "uc_p2p_bench runs device-initiated patterns only");
  if (pattern < UC_P2P_PINGPONG || pattern > UC_P2P_HALO) return fail(UC_ERR_ARG, "unknown pattern %d", pattern);
  if (bytes == 0 || bytes % 16) return fail(UC_ERR_ARG, "bytes must be a positive multiple of 16");
  if (iters < 1 || (pattern == UC_P2P_WINDOW && window < 1)) return fail(UC_ERR_ARG, "iters/window must be >= 1");
  if (sig->bytes < 8 * sizeof(uint64_t)) return fail(UC_ERR_ARG, "sig needs >= 8 u64");
  const size_t need = (pattern == UC_P2P_HALO ? 3 : 2) * bytes;
  if (buf->bytes < need) return fail(UC_ERR_ARG, "buf has %zu bytes, pattern needs %zu", buf->bytes, need);
  uc_comm* c = k->comm;
  UC_CUDA(cudaSetDevice(c->env->device));
  P2PLaunch L{};
  L.src = buf->local;
  L.sig_mine = (uint64_t*)sig->local;
  if (pattern == UC_P2P_HALO) {
    if (c->top >= 0) {
      L.dst_top = (char*)uc_mem_ptr(buf, c->top) + 2 * bytes;
      L.sig_top = (uint64_t*)uc_mem_ptr(sig, c->top);
    }
    if (c->bottom >= 0) {
      L.dst_bot = (char*)uc_mem_ptr(buf, c->bottom) + bytes;
      L.sig_bot = (uint64_t*)uc_mem_ptr(sig, c->bottom);
    }
    if ((c->top >= 0 && (!L.dst_top || !L.sig_top)) || (c->bottom >= 0 && (!L.dst_bot || !L.sig_bot)))
      return fail(UC_ERR_UNSUPPORTED, "a neighbour is not peer-addressable");
  } else {
    if (peer < 0 || peer >= c->size) return fail(UC_ERR_ARG, "peer %d out of range", peer);
    if (role != 0 && role != 1) return fail(UC_ERR_ARG, "role must be 0 or 1");
    L.dst_peer = (char*)uc_mem_ptr(buf, peer);
    L.sig_peer = (uint64_t*)uc_mem_ptr(sig, peer);
    if (!L.dst_peer || !L.sig_peer) return fail(UC_ERR_UNSUPPORTED, "rank %d not peer-addressable", peer);
    L.dst_peer = (char*)L.dst_peer + bytes;
  }
  L.bar = k->p2p_bar;
  L.bytes = bytes;
  // signal slots are disjoint per pattern (0: ping-pong, 1-2: window, 3-4: halo) and each
  // (pattern, peer) pair keeps its own monotone base, so partners only need to agree on the
  // calls they make together
  uint64_t& epoch = k->p2p_epoch[pattern][pattern == UC_P2P_HALO ? 0 : peer];
  L.base = epoch;
  L.iters = iters;
  L.window = pattern == UC_P2P_WINDOW ? window : 1;
  L.pattern = pattern;
  L.role = role;
  L.blocks = blocks;
  L.timeout_ns = k->timeout_ns;
  L.err = k->err;
  // every signal value of this call lies in (base, base + iters*window]; both partners advance alike
  epoch += (uint64_t)iters * (uint64_t)L.window + 1;
  return launch_p2p_bench(L, k->stream);
}

int uc_allreduce_sum(uc_coord* k, const void* send, void* recv, size_t count, uc_dtype dt) {
  return uc_allreduce(k, send, recv, count, dt, UC_SUM);  // collectives.cu
}

}  // extern "C"

int uc::oneshot_reduce(uc_coord* k, const void* send, void* recv, size_t count, uc_dtype dt, uc_redop op, int root) {
  if (dt != UC_F32 && dt != UC_F64 && dt != UC_U64) return fail(UC_ERR_ARG, "unknown dtype %d", (int)dt);
  uc_comm* c = k->comm;
  const size_t esz = dt == UC_F32 ? 4 : 8;
  if (count * esz > k->ar_slot_bytes)
    return fail(UC_ERR_UNSUPPORTED, "device-mode reductions support <= %zu bytes, got %zu", k->ar_slot_bytes,
                count * esz);
  const size_t P = (size_t)c->size;
  void* slots[UC_MAX_RANKS];
  uint64_t* flags[UC_MAX_RANKS];
  for (int q = 0; q < c->size; ++q) {
    char* base = (char*)uc_mem_ptr(k->ar_scratch, q);
    slots[q] = base;
    flags[q] = (uint64_t*)(base + 2 * P * k->ar_slot_bytes);
  }
  char* mine = (char*)k->ar_scratch->local;
  const uint64_t epoch = ++k->ar_epoch;
  return launch_allreduce_oneshot(send, recv, count, (int)dt, (int)op, root, c->rank, c->size, slots, flags,
                                  (const uint64_t*)(mine + 2 * P * k->ar_slot_bytes), mine, epoch, k->ar_slot_bytes,
                                  k->timeout_ns, k->err, k->stream);
}
