// merge.cu — multi-GPU merge of the per-rank tables (north_star subsystem 5): every table entry is a
// commutative fold (counters add, constant-bit masks AND), so ranks that consumed disjoint warp
// shards combine with ONE ncclAllReduce(sum, uint64) over a packed image in which each AND mask is
// byte-expanded (bit b -> byte b in {0,1}); after the sum a bit is set iff its byte == nranks
// (valid for nranks <= 255). A 2-word ncclMax allreduce of (checksum, ~checksum) proves that every
// rank registered the same sites (identical slot layout): with a host synchronisation the first
// time a context merges over a communicator, then checked on the device by the unpack kernel (no
// host round trip; a mismatch leaves the tables unmerged and sassi_read_tables reports EMISMATCH).
// sassi_merge_local runs the same pack / sum / unpack kernels for n contexts on one device, with
// the allreduce replaced by a device sum of their packed images.
// NCCL is loaded with dlopen (the torch-bundled libnccl.so.2 when already in the process).
#include <dlfcn.h>
#include <cstdlib>

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
    // the copy already in the process (torch loads its bundled NCCL), else the loader's search
    // path; SASSI_NCCL_LIB names another library explicitly
    const char* env = getenv("SASSI_NCCL_LIB");
    const char* names[] = {env ? env : "libnccl.so.2", "libnccl.so.2", "libnccl.so"};
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

// ck (optional): the (max checksum, max ~checksum) allreduce result; if it differs from this
// rank's checksum the ranks' layouts disagree: nothing is unpacked and err gets kMergeMismatch
__global__ void unpack_kernel(uint64_t* __restrict__ t, Offsets o, PackLayout L,
                              const uint64_t* __restrict__ pk, uint32_t nranks, const uint64_t* ck,
                              uint64_t checksum, uint32_t* err) {
  if (ck && (ck[0] != checksum || ~ck[1] != checksum)) {
    if (blockIdx.x == 0 && threadIdx.x == 0) atomicOr(err, kMergeMismatch);
    return;
  }
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

// sassi_merge_local's allreduce: sum of n packed images (the device copy of ncclAllReduce(sum))
__global__ void sum_packs_kernel(const uint64_t* const* __restrict__ packs, uint32_t n, uint64_t words,
                                 uint64_t* __restrict__ out) {
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < words; i += stride) {
    uint64_t v = 0;
    for (uint32_t r = 0; r < n; ++r) v += packs[r][i];
    out[i] = v;
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

int ensure_pack(sassi_ctx* c, const PackLayout& L) {
  if (L.total + 2 > c->pack_words) {
    cudaFree(c->d_pack);
    c->d_pack = nullptr;
    c->pack_words = 0;
    SASSI_CUDA(cudaMalloc(&c->d_pack, 8 * (L.total + 2)));
    c->pack_words = L.total + 2;
  }
  return SASSI_OK;
}

unsigned grid_for(uint64_t n) { return (unsigned)std::min<uint64_t>(4096, (n + 255) / 256); }

int ensure_dyn_gather(sassi_ctx* c, uint32_t nranks, uint32_t** gk, unsigned long long** gv) {
  const uint64_t cap = c->dyn_cap, kb = 4 * cap * nranks, vb = 8 * (2 * cap + 1) * nranks;
  const size_t need = ((kb + 255) & ~255ull) + vb;
  if (need > c->dyn_gather_bytes) {
    cudaFree(c->d_dyn_gather);
    c->d_dyn_gather = nullptr;
    c->dyn_gather_bytes = 0;
    SASSI_CUDA(cudaMalloc(&c->d_dyn_gather, need));
    c->dyn_gather_bytes = need;
  }
  *gk = static_cast<uint32_t*>(c->d_dyn_gather);
  *gv = reinterpret_cast<unsigned long long*>(static_cast<char*>(c->d_dyn_gather) + ((kb + 255) & ~255ull));
  return SASSI_OK;
}

// the gathered dynamic tables of all ranks re-inserted into this context's cleared table
int absorb_dyn(sassi_ctx* c, const uint32_t* gk, const unsigned long long* gv, uint32_t nranks,
               cudaStream_t s) {
  int rc = launch_dyn_reset(c, s);
  if (rc) return rc;
  dyn_absorb_kernel<<<grid_for((uint64_t)c->dyn_cap * nranks), 256, 0, s>>>(gk, gv, c->dyn_cap, nranks,
                                                                          c->d_dyn_keys, c->d_dyn_vals,
                                                                          c->dyn_lg);
  SASSI_CUDA(cudaGetLastError());
  c->launches += 1;
  return SASSI_OK;
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
  int rc = ensure_pack(c, L);
  if (rc) return rc;
  // 1) identical site tables on every rank? (max of (c, ~c) == (c, ~c) on every rank iff all equal)
  uint64_t* d_ck = c->d_pack + L.total;
  const uint64_t ck_host[2] = {c->checksum, ~c->checksum};
  SASSI_CUDA(cudaMemcpyAsync(d_ck, ck_host, 16, cudaMemcpyHostToDevice, s));
  r = N.AllReduce(d_ck, d_ck, 2, kNcclUint64, kNcclMax, comm, s);
  if (r) return nccl_err(r, "ncclAllReduce(checksum)");
  // The first merge of this context over this communicator (and every merge with dynamic pcs, whose
  // gather size depends on the configuration) waits for the verdict on the host before any
  // size-dependent collective. Afterwards the sizes cannot differ (sites and warps are fixed at
  // sassi_ctx_create) and the unpack kernel checks the checksum on the device: no host round trip.
  const bool sync_check = c->verified_comm != comm_v || c->verified_checksum != c->checksum || c->dyn_cap;
  if (sync_check) {
    uint64_t got[2];
    SASSI_CUDA(cudaMemcpyAsync(got, d_ck, 16, cudaMemcpyDeviceToHost, s));
    SASSI_CUDA(cudaStreamSynchronize(s));
    if (got[0] != c->checksum || ~got[1] != c->checksum)
      return set_error(SASSI_EMISMATCH, "site tables / n_warps / pc selection differ across ranks");
    c->verified_comm = comm_v;
    c->verified_checksum = c->checksum;
  }
  // 2) pack -> one allreduce(sum, u64) -> unpack
  pack_kernel<<<grid_for(L.total), 256, 0, s>>>(c->d_table, c->off, L, c->d_pack);
  SASSI_CUDA(cudaGetLastError());
  r = N.AllReduce(c->d_pack, c->d_pack, L.total, kNcclUint64, kNcclSum, comm, s);
  if (r) return nccl_err(r, "ncclAllReduce(tables)");
  unpack_kernel<<<grid_for(L.total), 256, 0, s>>>(c->d_table, c->off, L, c->d_pack, (uint32_t)nranks,
                                                  sync_check ? nullptr : d_ck, c->checksum, c->d_err);
  SASSI_CUDA(cudaGetLastError());
  c->launches += 2;
  // 3) dynamic pcs: slots differ across ranks (insertion order), so gather whole tables and rebuild
  if (c->dyn_cap) {
    uint32_t* gk;
    unsigned long long* gv;
    rc = ensure_dyn_gather(c, (uint32_t)nranks, &gk, &gv);
    if (rc) return rc;
    r = N.AllGather(c->d_dyn_keys, gk, c->dyn_cap, kNcclUint32, comm, s);
    if (r) return nccl_err(r, "ncclAllGather(dynamic keys)");
    r = N.AllGather(c->d_dyn_vals, gv, 2ull * c->dyn_cap + 1, kNcclUint64, comm, s);
    if (r) return nccl_err(r, "ncclAllGather(dynamic values)");
    rc = absorb_dyn(c, gk, gv, (uint32_t)nranks, s);
    if (rc) return rc;
  }
  return SASSI_OK;
}

// n contexts on one device: the same pack -> sum -> unpack, every context ends with the merge.
int launch_merge_local(sassi_ctx* const* ctxs, uint32_t n, cudaStream_t s) {
  sassi_ctx* c0 = ctxs[0];
  const PackLayout L = pack_layout(c0);
  for (uint32_t i = 0; i < n; ++i) {
    int rc = ensure_pack(ctxs[i], L);
    if (rc) return rc;
    pack_kernel<<<grid_for(L.total), 256, 0, s>>>(ctxs[i]->d_table, ctxs[i]->off, L, ctxs[i]->d_pack);
    SASSI_CUDA(cudaGetLastError());
    ctxs[i]->launches += 1;
  }
  // the sum goes to a scratch image (then every context unpacks it), pointers staged on the device
  uint64_t* d_sum = nullptr;
  const uint64_t** d_ptrs = nullptr;
  SASSI_CUDA(cudaMallocAsync(reinterpret_cast<void**>(&d_sum), 8 * L.total + 8 * n, s));
  d_ptrs = reinterpret_cast<const uint64_t**>(d_sum + L.total);
  std::vector<const uint64_t*> ptrs(n);
  for (uint32_t i = 0; i < n; ++i) ptrs[i] = ctxs[i]->d_pack;
  SASSI_CUDA(cudaMemcpyAsync(d_ptrs, ptrs.data(), 8 * n, cudaMemcpyHostToDevice, s));
  sum_packs_kernel<<<grid_for(L.total), 256, 0, s>>>(d_ptrs, n, L.total, d_sum);
  SASSI_CUDA(cudaGetLastError());
  for (uint32_t i = 0; i < n; ++i) {
    unpack_kernel<<<grid_for(L.total), 256, 0, s>>>(ctxs[i]->d_table, ctxs[i]->off, L, d_sum, n, nullptr,
                                                    0, nullptr);
    SASSI_CUDA(cudaGetLastError());
    ctxs[i]->launches += 1;
  }
  c0->launches += 1;
  // dynamic pcs: gather every context's table into c0's gather buffer, each context absorbs it
  if (c0->dyn_cap) {
    uint32_t* gk;
    unsigned long long* gv;
    int rc = ensure_dyn_gather(c0, n, &gk, &gv);
    if (rc) return rc;
    const uint64_t cap = c0->dyn_cap;
    for (uint32_t i = 0; i < n; ++i) {
      SASSI_CUDA(cudaMemcpyAsync(gk + cap * i, ctxs[i]->d_dyn_keys, 4 * cap, cudaMemcpyDeviceToDevice, s));
      SASSI_CUDA(cudaMemcpyAsync(gv + (2 * cap + 1) * i, ctxs[i]->d_dyn_vals, 8 * (2 * cap + 1),
                                 cudaMemcpyDeviceToDevice, s));
    }
    for (uint32_t i = 0; i < n; ++i) {
      rc = absorb_dyn(ctxs[i], gk, gv, n, s);
      if (rc) return rc;
    }
  }
  SASSI_CUDA(cudaFreeAsync(d_sum, s));
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
