// nccl_dyn.cu — NCCL for distributed contexts, resolved at run time with dlopen so that
// libdp binds to the NCCL the process already uses (torch's bundled libnccl.so.2) and loads
// without NCCL when it is not needed.  Per evaluation: one ncclReduceScatter of
// the WA gradient (nets are partitioned; each rank receives its cell block), one ncclAllReduce
// of the int64 bin map (P:253 step 1 summed over cell shards; exact), one of the WA partials
// (each slot nonzero on one rank only: exact) and one of the HPWL int64 limbs (exact, reading
// A7); the row-sharded Poisson solve adds a reduce-scatter of the map, two all-to-all
// transposes (grouped send / recv) and an all-gather of the field.
#include <dlfcn.h>

#include <cstring>

#include "dp_internal.h"

namespace dp {

namespace {

typedef struct { char internal[128]; } UniqueId;   // ncclUniqueId (NCCL_UNIQUE_ID_BYTES = 128)
typedef void *Comm;
typedef int Result;                                 // ncclResult_t, 0 = ncclSuccess
enum { kInt64 = 4, kUint64 = 5, kFloat32 = 7, kFloat64 = 8 };   // ncclDataType_t
enum { kSum = 0 };                                              // ncclRedOp_t

struct Api {
  void *handle = nullptr;
  Result (*get_unique_id)(UniqueId *) = nullptr;
  Result (*comm_init_rank)(Comm *, int, UniqueId, int) = nullptr;
  Result (*all_reduce)(const void *, void *, size_t, int, int, Comm, cudaStream_t) = nullptr;
  Result (*reduce_scatter)(const void *, void *, size_t, int, int, Comm, cudaStream_t) = nullptr;
  Result (*all_gather)(const void *, void *, size_t, int, Comm, cudaStream_t) = nullptr;
  Result (*send)(const void *, size_t, int, int, Comm, cudaStream_t) = nullptr;
  Result (*recv)(void *, size_t, int, int, Comm, cudaStream_t) = nullptr;
  Result (*group_start)() = nullptr;
  Result (*group_end)() = nullptr;
  Result (*comm_destroy)(Comm) = nullptr;
  const char *(*error_string)(Result) = nullptr;
};

Api g_api;

dp_status load() {
  if (g_api.handle) return DP_OK;
  void *h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_NOLOAD);
  if (!h) h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
  if (!h) h = dlopen("libnccl.so", RTLD_NOW | RTLD_GLOBAL);
  if (!h) return fail(DP_ERR_NCCL, std::string("cannot load NCCL: ") + dlerror());
  g_api.get_unique_id = (Result(*)(UniqueId *))dlsym(h, "ncclGetUniqueId");
  g_api.comm_init_rank = (Result(*)(Comm *, int, UniqueId, int))dlsym(h, "ncclCommInitRank");
  g_api.all_reduce = (Result(*)(const void *, void *, size_t, int, int, Comm, cudaStream_t))dlsym(h, "ncclAllReduce");
  g_api.comm_destroy = (Result(*)(Comm))dlsym(h, "ncclCommDestroy");
  g_api.reduce_scatter =
      (Result(*)(const void *, void *, size_t, int, int, Comm, cudaStream_t))dlsym(h, "ncclReduceScatter");
  g_api.all_gather = (Result(*)(const void *, void *, size_t, int, Comm, cudaStream_t))dlsym(h, "ncclAllGather");
  g_api.send = (Result(*)(const void *, size_t, int, int, Comm, cudaStream_t))dlsym(h, "ncclSend");
  g_api.recv = (Result(*)(void *, size_t, int, int, Comm, cudaStream_t))dlsym(h, "ncclRecv");
  g_api.group_start = (Result(*)())dlsym(h, "ncclGroupStart");
  g_api.group_end = (Result(*)())dlsym(h, "ncclGroupEnd");
  g_api.error_string = (const char *(*)(Result))dlsym(h, "ncclGetErrorString");
  if (!g_api.get_unique_id || !g_api.comm_init_rank || !g_api.all_reduce || !g_api.comm_destroy ||
      !g_api.reduce_scatter || !g_api.all_gather || !g_api.send || !g_api.recv || !g_api.group_start ||
      !g_api.group_end)
    return fail(DP_ERR_NCCL, "NCCL library lacks required symbols");
  g_api.handle = h;
  return DP_OK;
}

dp_status nccl_check(Result r, const char *what) {
  if (r == 0) return DP_OK;
  std::string msg = std::string("NCCL error in ") + what;
  if (g_api.error_string) msg += std::string(": ") + g_api.error_string(r);
  return fail(DP_ERR_NCCL, msg);
}

dp_status allreduce(Ctx &c, void *buf, size_t n, int dtype, cudaStream_t s) {
  if (!c.nccl_comm) return DP_OK;  // virtual shard: collectives skipped
  return nccl_check(g_api.all_reduce(buf, buf, n, dtype, kSum, (Comm)c.nccl_comm, s), "ncclAllReduce");
}

}  // namespace

dp_status nccl_get_unique_id(void *out128) {
  dp_status st = load();
  if (st != DP_OK) return st;
  UniqueId id;
  st = nccl_check(g_api.get_unique_id(&id), "ncclGetUniqueId");
  if (st != DP_OK) return st;
  std::memcpy(out128, id.internal, sizeof(id.internal));
  return DP_OK;
}

dp_status nccl_init(Ctx &c, const void *id) {
  dp_status st = load();
  if (st != DP_OK) return st;
  UniqueId uid;
  std::memcpy(uid.internal, id, sizeof(uid.internal));
  Comm comm = nullptr;
  st = nccl_check(g_api.comm_init_rank(&comm, c.world, uid, c.rank), "ncclCommInitRank");
  if (st != DP_OK) return st;
  c.nccl_comm = comm;
  return DP_OK;
}

dp_status nccl_allreduce_f32(Ctx &c, float *buf, size_t n, cudaStream_t s) { return allreduce(c, buf, n, kFloat32, s); }
dp_status nccl_allreduce_f64(Ctx &c, double *buf, size_t n, cudaStream_t s) { return allreduce(c, buf, n, kFloat64, s); }
dp_status nccl_allreduce_u64(Ctx &c, unsigned long long *buf, size_t n, cudaStream_t s) {
  return allreduce(c, buf, n, kUint64, s);
}

// in place: buf holds world blocks of n elements; this rank's block (buf + rank n) receives the sum
dp_status nccl_reduce_scatter(Ctx &c, void *buf, size_t n, int dtype, cudaStream_t s) {
  if (!c.nccl_comm) return DP_OK;
  const size_t esz = (dtype == kFloat32) ? 4 : 8;
  void *recv = static_cast<char *>(buf) + (size_t)c.rank * n * esz;
  return nccl_check(g_api.reduce_scatter(buf, recv, n, dtype, kSum, (Comm)c.nccl_comm, s), "ncclReduceScatter");
}
dp_status nccl_reduce_scatter_f32(Ctx &c, float *buf, size_t n, cudaStream_t s) {
  return nccl_reduce_scatter(c, buf, n, kFloat32, s);
}
dp_status nccl_reduce_scatter_i64(Ctx &c, long long *buf, size_t n, cudaStream_t s) {
  return nccl_reduce_scatter(c, buf, n, kInt64, s);
}
dp_status nccl_reduce_scatter_u64(Ctx &c, unsigned long long *buf, size_t n, cudaStream_t s) {
  return nccl_reduce_scatter(c, buf, n, kUint64, s);
}
// in place: this rank's block of n bytes at buf + rank n is gathered into every rank's buf
dp_status nccl_all_gather_bytes(Ctx &c, void *buf, size_t n, cudaStream_t s) {
  if (!c.nccl_comm) return DP_OK;
  const void *send = static_cast<const char *>(buf) + (size_t)c.rank * n;
  return nccl_check(g_api.all_gather(send, buf, n / 4, kFloat32, (Comm)c.nccl_comm, s), "ncclAllGather");
}
// all-to-all of equal byte blocks: block q of send goes to rank q, block r of recv comes from rank r
dp_status nccl_all_to_all_bytes(Ctx &c, const void *send, void *recv, size_t n, cudaStream_t s) {
  if (!c.nccl_comm) return DP_OK;
  dp_status st = nccl_check(g_api.group_start(), "ncclGroupStart");
  if (st != DP_OK) return st;
  for (int q = 0; q < c.world && st == DP_OK; q++) {
    st = nccl_check(g_api.send(static_cast<const char *>(send) + (size_t)q * n, n / 4, kFloat32, q,
                               (Comm)c.nccl_comm, s), "ncclSend");
    if (st == DP_OK)
      st = nccl_check(g_api.recv(static_cast<char *>(recv) + (size_t)q * n, n / 4, kFloat32, q, (Comm)c.nccl_comm, s),
                      "ncclRecv");
  }
  const dp_status st2 = nccl_check(g_api.group_end(), "ncclGroupEnd");
  return st != DP_OK ? st : st2;
}

void nccl_destroy(Ctx &c) {
  if (c.nccl_comm && g_api.comm_destroy) g_api.comm_destroy((Comm)c.nccl_comm);
  c.nccl_comm = nullptr;
}

}  // namespace dp
