// merge.cu — multi-GPU merge of the per-rank tables (north_star subsystem 5): every table entry is a
// commutative fold (counters add, constant-bit masks AND), so ranks that consumed disjoint warp
// shards combine with ONE ncclAllReduce(sum, uint64) over a packed image in which each AND mask is
// byte-expanded (bit b -> byte b in {0,1}); after the sum a bit is set iff its byte == nranks
// (valid for nranks <= 255). A tiny ncclMax allreduce of (checksum, ~checksum) first proves that
// every rank registered the same sites (identical slot layout).
// NCCL is loaded with dlopen (the torch-bundled libnccl.so.2 when already in the process).
#include <dlfcn.h>

#include <mutex>

#include "common.cuh"

namespace sassi {
namespace {

// minimal NCCL ABI (nccl.h 2.x)
typedef struct ncclComm* ncclComm_t;
typedef struct {
  char internal[128];
} ncclUniqueId;
typedef int ncclResult_t;
enum { kNcclUint32 = 3, kNcclUint64 = 5 };
enum { kNcclSum = 0, kNcclMax = 2 };

struct Nccl {
  ncclResult_t (*GetUniqueId)(ncclUniqueId*) = nullptr;
  ncclResult_t (*CommInitRank)(ncclComm_t*, int, ncclUniqueId, int) = nullptr;
  ncclResult_t (*CommDestroy)(ncclComm_t) = nullptr;
  ncclResult_t (*CommCount)(const ncclComm_t, int*) = nullptr;
  ncclResult_t (*AllReduce)(const void*, void*, size_t, int, int, ncclComm_t, cudaStream_t) = nullptr;
  ncclResult_t (*AllGather)(const void*, void*, size_t, int, ncclComm_t, cudaStream_t) = nullptr;
  const char* (*GetErrorString)(ncclResult_t) = nullptr;
  bool ok = false;
  std::string why;
};

Nccl& nccl() {
  static Nccl n;
  static std::once_flag once;
  std::call_once(once, [] {
    const char* names[] = {"libnccl.so.2", "libnccl.so",
                           "/opt/prime-rl/.venv/lib/python3.12/site-packages/nvidia/nccl/lib/libnccl.so.2"};
    void* h = nullptr;
    for (const char* nm : names) {
      h = dlopen(nm, RTLD_NOW | RTLD_NOLOAD | RTLD_GLOBAL);  // prefer the copy already loaded
      if (h) break;
    }
    for (const char* nm : names) {
      if (h) break;
      h = dlopen(nm, RTLD_NOW | RTLD_GLOBAL);
    }
    if (!h) {
      n.why = "cannot dlopen libnccl.so.2";
      return;
    }
    n.GetUniqueId = (decltype(n.GetUniqueId))dlsym(h, "ncclGetUniqueId");
    n.CommInitRank = (decltype(n.CommInitRank))dlsym(h, "ncclCommInitRank");
    n.CommDestroy = (decltype(n.CommDestroy))dlsym(h, "ncclCommDestroy");
    n.CommCount = (decltype(n.CommCount))dlsym(h, "ncclCommCount");
    n.AllReduce = (decltype(n.AllReduce))dlsym(h, "ncclAllReduce");
    n.AllGather = (decltype(n.AllGather))dlsym(h, "ncclAllGather");
    n.GetErrorString = (decltype(n.GetErrorString))dlsym(h, "ncclGetErrorString");
    n.ok = n.GetUniqueId && n.CommInitRank && n.CommDestroy && n.CommCount && n.AllReduce &&
           n.AllGather && n.GetErrorString;
    if (!n.ok) n.why = "libnccl.so.2 lacks an expected symbol";
  });
  return n;
}

int nccl_err(ncclResult_t r, const char* what) {
  return set_error(SASSI_ENCCL, std::string(what) + ": " + nccl().GetErrorString(r));
}

// packed image: [4 diag][br..val sums][h32..imix sums, then pcmat sums][isScalar 0/1 sums, 4S]
// [ones+zeros masks byte-expanded, 8S x 4 words]. After the sum: isScalar = (sum == nranks); mask
// bit set iff its byte == nranks. pcsel (configuration, equal on every rank) is not packed.
struct PackLayout {
  uint64_t n_sum_a, n_sum_b1, n_sum_b, n_scalar, n_mask_words, total;
};
PackLayout pack_layout(const sassi_ctx* c) {
  PackLayout L;
  L.n_sum_a = c->off.ones - c->off.br;
  L.n_sum_b1 = c->off.pcsel - c->off.h32;
  L.n_sum_b = L.n_sum_b1 + (c->off.total - c->off.pcmat);
  L.n_scalar = 4ull * c->S;
  L.n_mask_words = 8ull * c->S * 4;
  L.total = 4 + L.n_sum_a + L.n_sum_b + L.n_scalar + L.n_mask_words;
  return L;
}

__global__ void pack_kernel(const uint64_t* __restrict__ t, Offsets o, PackLayout L, uint64_t* pk) {
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  const uint64_t b1 = 4 + L.n_sum_a, b2 = b1 + L.n_sum_b, b3 = b2 + L.n_scalar;
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < L.total; i += stride) {
    uint64_t v;
    if (i < 4) v = t[i];
    else if (i < b1) v = t[o.br + (i - 4)];
    else if (i < b1 + L.n_sum_b1) v = t[o.h32 + (i - b1)];
    else if (i < b2) v = t[o.pcmat + (i - b1 - L.n_sum_b1)];
    else if (i < b3) v = t[o.scalar + (i - b2)];
    else {
      const uint64_t w = i - b3;
      const uint32_t mask = (uint32_t)t[o.ones + w / 4];  // ones[S][4] then zeros[S][4]
      const uint32_t byte8 = (mask >> (8 * (w % 4))) & 0xFFu;
      v = 0;
#pragma unroll
      for (int b = 0; b < 8; ++b) v |= (uint64_t)((byte8 >> b) & 1u) << (8 * b);
    }
    pk[i] = v;
  }
}

__global__ void unpack_kernel(uint64_t* __restrict__ t, Offsets o, PackLayout L,
                              const uint64_t* __restrict__ pk, uint32_t nranks) {
  const uint64_t b1 = 4 + L.n_sum_a, b2 = b1 + L.n_sum_b, b3 = b2 + L.n_scalar;
  const uint64_t n_items = b3 + L.n_mask_words / 4;
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n_items; i += stride) {
    if (i < 4) t[i] = pk[i];
    else if (i < b1) t[o.br + (i - 4)] = pk[i];
    else if (i < b1 + L.n_sum_b1) t[o.h32 + (i - b1)] = pk[i];
    else if (i < b2) t[o.pcmat + (i - b1 - L.n_sum_b1)] = pk[i];
    else if (i < b3) t[o.scalar + (i - b2)] = pk[i] == nranks ? 1ull : 0ull;
    else {
      const uint64_t m = i - b3;
      const uint64_t* w = pk + b3 + 4 * m;
      uint32_t mask = 0;
      for (int q = 0; q < 4; ++q)
        for (int b = 0; b < 8; ++b)
          if (((w[q] >> (8 * b)) & 0xFFu) == nranks) mask |= 1u << (8 * q + b);
      t[o.ones + m] = mask;
    }
  }
}

// dynamic tables: every rank's (keys, values) gathered; re-insert all of them into the cleared
// local table (one thread per gathered slot), dropped records summed
__global__ void dyn_absorb_kernel(const uint32_t* __restrict__ gk, const unsigned long long* __restrict__ gv,
                                  uint32_t cap, uint32_t nranks, uint32_t* keys, unsigned long long* vals,
                                  uint32_t lg) {
  const uint64_t n = (uint64_t)cap * nranks;
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x) {
    const uint32_t r = (uint32_t)(i / cap), slot = (uint32_t)(i % cap);
    const unsigned long long* v = gv + (2ull * cap + 1) * r;
    if (slot == 0 && v[2ull * cap]) atomicAdd(vals + 2ull * cap, v[2ull * cap]);
    const uint32_t k = gk[i];
    if (k != EMPTY_KEY) dyn_insert(k, v[2ull * slot], v[2ull * slot + 1], keys, vals, cap, lg);
  }
}

}  // namespace

int launch_merge(sassi_ctx* c, void* comm_v, cudaStream_t s) {
  Nccl& N = nccl();
  if (!N.ok) return set_error(SASSI_ENCCL, N.why);
  ncclComm_t comm = (ncclComm_t)comm_v;
  int nranks = 0;
  ncclResult_t r = N.CommCount(comm, &nranks);
  if (r) return nccl_err(r, "ncclCommCount");
  if (nranks > 255) return set_error(SASSI_EINVAL, "sassi_merge supports at most 255 ranks");
  const PackLayout L = pack_layout(c);
  if (L.total + 2 > c->pack_words) {
    cudaFree(c->d_pack);
    c->d_pack = nullptr;
    c->pack_words = 0;
    SASSI_CUDA(cudaMalloc(&c->d_pack, 8 * (L.total + 2)));
    c->pack_words = L.total + 2;
  }
  // 1) identical site tables on every rank?
  uint64_t ck[2] = {c->checksum, ~c->checksum};
  uint64_t* d_ck = c->d_pack + L.total;
  SASSI_CUDA(cudaMemcpyAsync(d_ck, ck, 16, cudaMemcpyHostToDevice, s));
  r = N.AllReduce(d_ck, d_ck, 2, kNcclUint64, kNcclMax, comm, s);
  if (r) return nccl_err(r, "ncclAllReduce(checksum)");
  uint64_t got[2];
  SASSI_CUDA(cudaMemcpyAsync(got, d_ck, 16, cudaMemcpyDeviceToHost, s));
  SASSI_CUDA(cudaStreamSynchronize(s));
  if (got[0] != c->checksum || ~got[1] != c->checksum)
    return set_error(SASSI_EMISMATCH, "site tables / n_warps differ across ranks");
  // 2) pack -> one allreduce(sum, u64) -> unpack
  const unsigned grid = (unsigned)std::min<uint64_t>(4096, (L.total + 255) / 256);
  pack_kernel<<<grid, 256, 0, s>>>(c->d_table, c->off, L, c->d_pack);
  SASSI_CUDA(cudaGetLastError());
  r = N.AllReduce(c->d_pack, c->d_pack, L.total, kNcclUint64, kNcclSum, comm, s);
  if (r) return nccl_err(r, "ncclAllReduce(tables)");
  unpack_kernel<<<grid, 256, 0, s>>>(c->d_table, c->off, L, c->d_pack, (uint32_t)nranks);
  SASSI_CUDA(cudaGetLastError());
  c->launches += 2;
  // 3) dynamic pcs: slots differ across ranks (insertion order), so gather whole tables and rebuild
  if (c->dyn_cap) {
    const uint64_t cap = c->dyn_cap, kb = 4 * cap * nranks, vb = 8 * (2 * cap + 1) * nranks;
    const size_t need = ((kb + 255) & ~255ull) + vb;
    if (need > c->dyn_gather_bytes) {
      cudaFree(c->d_dyn_gather);
      c->d_dyn_gather = nullptr;
      c->dyn_gather_bytes = 0;
      SASSI_CUDA(cudaMalloc(&c->d_dyn_gather, need));
      c->dyn_gather_bytes = need;
    }
    uint32_t* gk = static_cast<uint32_t*>(c->d_dyn_gather);
    unsigned long long* gv = reinterpret_cast<unsigned long long*>(static_cast<char*>(c->d_dyn_gather) +
                                                                   ((kb + 255) & ~255ull));
    r = N.AllGather(c->d_dyn_keys, gk, cap, kNcclUint32, comm, s);
    if (r) return nccl_err(r, "ncclAllGather(dynamic keys)");
    r = N.AllGather(c->d_dyn_vals, gv, 2 * cap + 1, kNcclUint64, comm, s);
    if (r) return nccl_err(r, "ncclAllGather(dynamic values)");
    int rc = launch_dyn_reset(c, s);
    if (rc) return rc;
    const unsigned g2 = (unsigned)std::min<uint64_t>(4096, (cap * nranks + 255) / 256);
    dyn_absorb_kernel<<<g2, 256, 0, s>>>(gk, gv, c->dyn_cap, (uint32_t)nranks, c->d_dyn_keys,
                                         c->d_dyn_vals, c->dyn_lg);
    SASSI_CUDA(cudaGetLastError());
    c->launches += 1;
  }
  return SASSI_OK;
}

}  // namespace sassi

extern "C" {

int sassi_nccl_get_unique_id(void* out) {
  using namespace sassi;
  if (!out) return set_error(SASSI_EINVAL, "null out");
  Nccl& N = nccl();
  if (!N.ok) return set_error(SASSI_ENCCL, N.why);
  ncclUniqueId id;
  ncclResult_t r = N.GetUniqueId(&id);
  if (r) return nccl_err(r, "ncclGetUniqueId");
  memcpy(out, &id, sizeof id);
  return SASSI_OK;
}

int sassi_nccl_comm_create(void** comm_out, int nranks, int rank, const void* uid, int device) {
  using namespace sassi;
  if (!comm_out || !uid) return set_error(SASSI_EINVAL, "null argument");
  Nccl& N = nccl();
  if (!N.ok) return set_error(SASSI_ENCCL, N.why);
  SASSI_CUDA(cudaSetDevice(device));
  ncclUniqueId id;
  memcpy(&id, uid, sizeof id);
  ncclComm_t comm = nullptr;
  ncclResult_t r = N.CommInitRank(&comm, nranks, id, rank);
  if (r) return nccl_err(r, "ncclCommInitRank");
  *comm_out = comm;
  return SASSI_OK;
}

int sassi_nccl_comm_destroy(void* comm) {
  using namespace sassi;
  if (!comm) return SASSI_OK;
  Nccl& N = nccl();
  if (!N.ok) return set_error(SASSI_ENCCL, N.why);
  ncclResult_t r = N.CommDestroy((ncclComm_t)comm);
  if (r) return nccl_err(r, "ncclCommDestroy");
  return SASSI_OK;
}

}  // extern "C"
