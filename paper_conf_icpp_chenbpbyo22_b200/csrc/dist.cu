// dist.cu -- partition construction and the exchange layer of the
// partitioned BFS / PageRank path (S10):
//   * loopback: P partitions of one graph on one device in one process; the
//     exchange is device-to-device copies (tests the whole protocol on 1 GPU);
//   * NCCL: one partition per process (torchrun), grouped ncclSend/ncclRecv
//     for the per-destination counts and payloads, ncclAllReduce for the
//     global termination test.  NCCL is resolved with dlopen("libnccl.so.2")
//     at first use, so the library carries no link-time NCCL dependency.
#include <dlfcn.h>
#include <nccl.h>

#include <algorithm>
#include <cstring>
#include <mutex>
#include <vector>

#include "internal.h"

namespace atos {

int upload_part_local(Part& p, const int64_t* row_ptr, const int32_t* col, int where, int64_t nl, int64_t ml);

// ------------------------------------------------------------ NCCL (dlopen)
namespace {
struct NcclApi {
  bool ok = false;
  ncclResult_t (*GetUniqueId)(ncclUniqueId*) = nullptr;
  ncclResult_t (*CommInitRank)(ncclComm_t*, int, ncclUniqueId, int) = nullptr;
  ncclResult_t (*CommDestroy)(ncclComm_t) = nullptr;
  ncclResult_t (*Send)(const void*, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t) = nullptr;
  ncclResult_t (*Recv)(void*, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t) = nullptr;
  ncclResult_t (*GroupStart)() = nullptr;
  ncclResult_t (*GroupEnd)() = nullptr;
  ncclResult_t (*AllReduce)(const void*, void*, size_t, ncclDataType_t, ncclRedOp_t, ncclComm_t,
                            cudaStream_t) = nullptr;
  const char* (*GetErrorString)(ncclResult_t) = nullptr;
};

NcclApi& nccl() {
  static NcclApi api;
  static std::once_flag once;
  std::call_once(once, [] {
    void* h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
    if (!h) h = dlopen("libnccl.so", RTLD_NOW | RTLD_GLOBAL);
    if (!h) return;
#define SYM(f) api.f = (decltype(api.f))dlsym(h, "nccl" #f)
    SYM(GetUniqueId);
    SYM(CommInitRank);
    SYM(CommDestroy);
    SYM(Send);
    SYM(Recv);
    SYM(GroupStart);
    SYM(GroupEnd);
    SYM(AllReduce);
    SYM(GetErrorString);
#undef SYM
    api.ok = api.GetUniqueId && api.CommInitRank && api.CommDestroy && api.Send && api.Recv && api.GroupStart &&
             api.GroupEnd && api.AllReduce && api.GetErrorString;
  });
  return api;
}
}  // namespace

#define ATOS_NCCL(call)                                                                        \
  do {                                                                                        \
    ncclResult_t e_ = (call);                                                                 \
    if (e_ != ncclSuccess) {                                                                  \
      set_error("%s failed: %s (%s:%d)", #call, nccl().GetErrorString(e_), __FILE__, __LINE__); \
      return ATOS_ERR_NCCL;                                                                   \
    }                                                                                         \
  } while (0)

// --------------------------------------------------------------- exchanges
int exchange_loopback(std::vector<ExchangeIO>& io, size_t val_bytes, cudaStream_t s) {
  const size_t P = io.size();
  for (size_t d = 0; d < P; ++d) {
    uint64_t total = 0;
    for (size_t src = 0; src < P; ++src) total += io[src].counts[d];
    io[d].in_total = total;
    ATOS_TRY(io[d].in_vid->ensure(std::max<uint64_t>(total, 1) * 4));
    ATOS_TRY(io[d].in_val->ensure(std::max<uint64_t>(total, 1) * val_bytes));
  }
  for (size_t src = 0; src < P; ++src) {
    uint64_t seg = 0;
    for (size_t d = 0; d < P; ++d) {
      const uint64_t c = io[src].counts[d];
      if (c) {
        // offset of src's segment inside d's inbox
        uint64_t off = 0;
        for (size_t s2 = 0; s2 < src; ++s2) off += io[s2].counts[d];
        ATOS_CUDA(cudaMemcpyAsync(io[d].in_vid->as<uint32_t>() + off, io[src].out_vid + seg, c * 4,
                                  cudaMemcpyDeviceToDevice, s));
        ATOS_CUDA(cudaMemcpyAsync((char*)io[d].in_val->p + off * val_bytes,
                                  (const char*)io[src].out_val + seg * val_bytes, c * val_bytes,
                                  cudaMemcpyDeviceToDevice, s));
      }
      seg += c;
    }
  }
  return ATOS_OK;
}

// Host-staged exchange (atos_comm_create_host): the same two steps as the NCCL path -- per-destination
// counts, then the SoA payloads -- but through the caller's host alltoallv (e.g. torch.distributed gloo).
// Each peer's message is [ids: c x u32][values: c x val_bytes].
static int exchange_host(Comm* c, ExchangeIO& io, size_t val_bytes, cudaStream_t s, uint64_t* bytes_sent) {
  const int P = c->nranks;
  std::vector<uint64_t> cb(P, 8), rcnt(P, 0);
  if (c->h_a2a(c->h_user, io.counts.data(), cb.data(), rcnt.data(), cb.data()) != 0) {
    set_error("host alltoallv (counts) failed");
    return ATOS_ERR_NCCL;
  }
  uint64_t stot = 0, rtot = 0;
  for (int p = 0; p < P; ++p) {
    stot += io.counts[p];
    rtot += rcnt[p];
  }
  const size_t item = 4 + val_bytes;
  std::vector<char> sbuf(std::max<uint64_t>(stot, 1) * item), rbuf(std::max<uint64_t>(rtot, 1) * item);
  std::vector<uint32_t> ids(std::max<uint64_t>(stot, 1));
  std::vector<char> vals(std::max<uint64_t>(stot, 1) * val_bytes);
  if (stot) {
    ATOS_CUDA(cudaMemcpyAsync(ids.data(), io.out_vid, stot * 4, cudaMemcpyDeviceToHost, s));
    ATOS_CUDA(cudaMemcpyAsync(vals.data(), io.out_val, stot * val_bytes, cudaMemcpyDeviceToHost, s));
  }
  ATOS_CUDA(cudaStreamSynchronize(s));
  std::vector<uint64_t> sb(P), rb(P);
  uint64_t so = 0, b = 0;
  char* w = sbuf.data();
  for (int p = 0; p < P; ++p) {
    const uint64_t k = io.counts[p];
    memcpy(w, ids.data() + so, k * 4);
    memcpy(w + k * 4, vals.data() + so * val_bytes, k * val_bytes);
    w += k * item;
    so += k;
    sb[p] = k * item;
    rb[p] = rcnt[p] * item;
    if (p != c->rank) b += k * item;
  }
  if (c->h_a2a(c->h_user, sbuf.data(), sb.data(), rbuf.data(), rb.data()) != 0) {
    set_error("host alltoallv (payload) failed");
    return ATOS_ERR_NCCL;
  }
  io.in_total = rtot;
  ATOS_TRY(io.in_vid->ensure(std::max<uint64_t>(rtot, 1) * 4));
  ATOS_TRY(io.in_val->ensure(std::max<uint64_t>(rtot, 1) * val_bytes));
  std::vector<uint32_t> rid(std::max<uint64_t>(rtot, 1));
  std::vector<char> rval(std::max<uint64_t>(rtot, 1) * val_bytes);
  const char* q = rbuf.data();
  uint64_t ro = 0;
  for (int p = 0; p < P; ++p) {
    const uint64_t k = rcnt[p];
    memcpy(rid.data() + ro, q, k * 4);
    memcpy(rval.data() + ro * val_bytes, q + k * 4, k * val_bytes);
    q += k * item;
    ro += k;
  }
  if (rtot) {
    ATOS_CUDA(cudaMemcpyAsync(io.in_vid->p, rid.data(), rtot * 4, cudaMemcpyHostToDevice, s));
    ATOS_CUDA(cudaMemcpyAsync(io.in_val->p, rval.data(), rtot * val_bytes, cudaMemcpyHostToDevice, s));
  }
  ATOS_CUDA(cudaStreamSynchronize(s));  // the host vectors die at return
  if (bytes_sent) *bytes_sent = b;
  return ATOS_OK;
}

int exchange_nccl(Comm* c, ExchangeIO& io, size_t val_bytes, cudaStream_t s, uint64_t* bytes_sent) {
  if (c->h_a2a) return exchange_host(c, io, val_bytes, s, bytes_sent);
  NcclApi& api = nccl();
  const int P = c->nranks;
  ncclComm_t comm = (ncclComm_t)c->nccl;
  // 1. counts: P u64 out, P u64 in (device staging in the inbox buffers' scratch)
  static thread_local DevBuf cbuf;
  ATOS_TRY(cbuf.ensure(sizeof(uint64_t) * 2 * P));
  uint64_t* d_send = cbuf.as<uint64_t>();
  uint64_t* d_recv = d_send + P;
  ATOS_CUDA(cudaMemcpyAsync(d_send, io.counts.data(), sizeof(uint64_t) * P, cudaMemcpyHostToDevice, s));
  ATOS_NCCL(api.GroupStart());
  for (int p = 0; p < P; ++p) {
    ATOS_NCCL(api.Send(d_send + p, 1, ncclUint64, p, comm, s));
    ATOS_NCCL(api.Recv(d_recv + p, 1, ncclUint64, p, comm, s));
  }
  ATOS_NCCL(api.GroupEnd());
  std::vector<uint64_t> rc(P);
  ATOS_CUDA(cudaMemcpyAsync(rc.data(), d_recv, sizeof(uint64_t) * P, cudaMemcpyDeviceToHost, s));
  ATOS_CUDA(cudaStreamSynchronize(s));
  uint64_t total = 0;
  for (int p = 0; p < P; ++p) total += rc[p];
  io.in_total = total;
  ATOS_TRY(io.in_vid->ensure(std::max<uint64_t>(total, 1) * 4));
  ATOS_TRY(io.in_val->ensure(std::max<uint64_t>(total, 1) * val_bytes));
  // 2. payloads (SoA: ids then values), one grouped round of sends/recvs
  ATOS_NCCL(api.GroupStart());
  uint64_t so = 0, ro = 0, b = 0;
  for (int p = 0; p < P; ++p) {
    if (io.counts[p]) {
      ATOS_NCCL(api.Send(io.out_vid + so, io.counts[p], ncclUint32, p, comm, s));
      ATOS_NCCL(api.Send((const char*)io.out_val + so * val_bytes, io.counts[p] * val_bytes, ncclUint8, p, comm, s));
      if (p != c->rank) b += io.counts[p] * (4 + val_bytes);
    }
    if (rc[p]) {
      ATOS_NCCL(api.Recv(io.in_vid->as<uint32_t>() + ro, rc[p], ncclUint32, p, comm, s));
      ATOS_NCCL(api.Recv((char*)io.in_val->p + ro * val_bytes, rc[p] * val_bytes, ncclUint8, p, comm, s));
    }
    so += io.counts[p];
    ro += rc[p];
  }
  ATOS_NCCL(api.GroupEnd());
  if (bytes_sent) *bytes_sent = b;
  return ATOS_OK;
}

int allreduce_u64(Comm* c, uint64_t* v, cudaStream_t s) {
  if (c->h_ar) {
    ATOS_CUDA(cudaStreamSynchronize(s));
    if (c->h_ar(c->h_user, v, 0) != 0) {
      set_error("host allreduce (u64) failed");
      return ATOS_ERR_NCCL;
    }
    return ATOS_OK;
  }
  static thread_local DevBuf buf;
  ATOS_TRY(buf.ensure(8));
  ATOS_CUDA(cudaMemcpyAsync(buf.p, v, 8, cudaMemcpyHostToDevice, s));
  ATOS_NCCL(nccl().AllReduce(buf.p, buf.p, 1, ncclUint64, ncclSum, (ncclComm_t)c->nccl, s));
  ATOS_CUDA(cudaMemcpyAsync(v, buf.p, 8, cudaMemcpyDeviceToHost, s));
  ATOS_CUDA(cudaStreamSynchronize(s));
  return ATOS_OK;
}

int allgather_host(Comm* c, const void* in, size_t bytes, void* out, cudaStream_t s) {
  const int P = c->nranks;
  if (c->h_a2a) {
    std::vector<char> sbuf((size_t)P * bytes);
    for (int p = 0; p < P; ++p) memcpy(sbuf.data() + (size_t)p * bytes, in, bytes);
    std::vector<uint64_t> cnt(P, bytes);
    if (c->h_a2a(c->h_user, sbuf.data(), cnt.data(), out, cnt.data()) != 0) {
      set_error("host alltoallv (allgather) failed");
      return ATOS_ERR_NCCL;
    }
    return ATOS_OK;
  }
  static thread_local DevBuf buf;
  ATOS_TRY(buf.ensure((size_t)P * bytes * 2));
  char* d_in = buf.as<char>();
  char* d_out = d_in + (size_t)P * bytes;
  ATOS_CUDA(cudaMemcpyAsync(d_in, in, bytes, cudaMemcpyHostToDevice, s));
  NcclApi& api = nccl();
  ATOS_NCCL(api.GroupStart());
  for (int p = 0; p < P; ++p) {
    ATOS_NCCL(api.Send(d_in, bytes, ncclUint8, p, (ncclComm_t)c->nccl, s));
    ATOS_NCCL(api.Recv(d_out + (size_t)p * bytes, bytes, ncclUint8, p, (ncclComm_t)c->nccl, s));
  }
  ATOS_NCCL(api.GroupEnd());
  ATOS_CUDA(cudaMemcpyAsync(out, d_out, (size_t)P * bytes, cudaMemcpyDeviceToHost, s));
  ATOS_CUDA(cudaStreamSynchronize(s));
  return ATOS_OK;
}

int allreduce_f64(Comm* c, double* v, cudaStream_t s) {
  if (c->h_ar) {
    ATOS_CUDA(cudaStreamSynchronize(s));
    if (c->h_ar(c->h_user, v, 1) != 0) {
      set_error("host allreduce (f64) failed");
      return ATOS_ERR_NCCL;
    }
    return ATOS_OK;
  }
  static thread_local DevBuf buf;
  ATOS_TRY(buf.ensure(8));
  ATOS_CUDA(cudaMemcpyAsync(buf.p, v, 8, cudaMemcpyHostToDevice, s));
  ATOS_NCCL(nccl().AllReduce(buf.p, buf.p, 1, ncclFloat64, ncclSum, (ncclComm_t)c->nccl, s));
  ATOS_CUDA(cudaMemcpyAsync(v, buf.p, 8, cudaMemcpyDeviceToHost, s));
  ATOS_CUDA(cudaStreamSynchronize(s));
  return ATOS_OK;
}

// ----------------------------------------------------- partition creation
int create_loopback_parts(atos_csr* g, const int64_t* row_ptr, const int32_t* col, int where) {
  const int P = g->num_parts;
  g->parts.resize(P);
  for (int p = 0; p < P; ++p) {
    int64_t vb = 0, ve = 0;
    atos_partition_range(g->n, P, p, &vb, &ve);
    int64_t eb = 0, ee = 0;
    if (where == ATOS_MEM_HOST) {
      eb = row_ptr[vb];
      ee = row_ptr[ve];
    } else {
      ATOS_CUDA(cudaMemcpy(&eb, row_ptr + vb, 8, cudaMemcpyDeviceToHost));
      ATOS_CUDA(cudaMemcpy(&ee, row_ptr + ve, 8, cudaMemcpyDeviceToHost));
    }
    Part& part = g->parts[p];
    ATOS_TRY(upload_part_local(part, row_ptr + vb, col + eb, where, ve - vb, ee - eb));
    // rebase: upload_part_local expects offsets relative to row_ptr[vb]
    part.v_begin = vb;
    part.v_end = ve;
  }
  return ATOS_OK;
}

}  // namespace atos

using namespace atos;

struct atos_comm {
  Comm c;
};

extern "C" {

int atos_comm_unique_id(void* id_out, size_t len) {
  if (!id_out || len < sizeof(ncclUniqueId)) {
    set_error("atos_comm_unique_id: need a buffer of %zu bytes", sizeof(ncclUniqueId));
    return ATOS_ERR_INVALID_ARG;
  }
  if (!nccl().ok) {
    set_error("atos_comm_unique_id: libnccl.so.2 could not be loaded");
    return ATOS_ERR_NCCL;
  }
  ncclUniqueId id;
  ATOS_NCCL(nccl().GetUniqueId(&id));
  memcpy(id_out, &id, sizeof(id));
  return ATOS_OK;
}

int atos_comm_create(atos_comm** out, int nranks, int rank, const void* id, size_t len, int device) {
  if (!out || nranks < 1 || rank < 0 || rank >= nranks || !id || len < sizeof(ncclUniqueId)) {
    set_error("atos_comm_create: invalid argument");
    return ATOS_ERR_INVALID_ARG;
  }
  *out = nullptr;
  if (!nccl().ok) {
    set_error("atos_comm_create: libnccl.so.2 could not be loaded");
    return ATOS_ERR_NCCL;
  }
  DeviceGuard dg(device);
  ncclUniqueId uid;
  memcpy(&uid, id, sizeof(uid));
  ncclComm_t comm = nullptr;
  ATOS_NCCL(nccl().CommInitRank(&comm, nranks, uid, rank));
  atos_comm* c = new atos_comm();
  c->c.nranks = nranks;
  c->c.rank = rank;
  c->c.device = device;
  c->c.nccl = comm;
  *out = c;
  return ATOS_OK;
}

int atos_comm_create_host(atos_comm** out, int nranks, int rank, int device, atos_host_alltoallv_fn alltoallv,
                          atos_host_allreduce_fn allreduce, void* user) {
  if (!out || nranks < 1 || rank < 0 || rank >= nranks || !alltoallv || !allreduce) {
    set_error("atos_comm_create_host: invalid argument");
    return ATOS_ERR_INVALID_ARG;
  }
  int ndev = 0;
  if (cudaGetDeviceCount(&ndev) != cudaSuccess || device < 0 || device >= ndev) {
    cudaGetLastError();
    set_error("atos_comm_create_host: device %d not available", device);
    return ATOS_ERR_CUDA;
  }
  atos_comm* c = new atos_comm();
  c->c.nranks = nranks;
  c->c.rank = rank;
  c->c.device = device;
  c->c.h_a2a = alltoallv;
  c->c.h_ar = allreduce;
  c->c.h_user = user;
  *out = c;
  return ATOS_OK;
}

void atos_comm_destroy(atos_comm* c) {
  if (!c) return;
  if (c->c.nccl && nccl().ok) nccl().CommDestroy((ncclComm_t)c->c.nccl);
  delete c;
}

int atos_comm_gather(atos_comm* comm, int64_t n_global, const void* slice, size_t elem_bytes, void* out_root,
                     void* stream) {
  if (!comm || n_global < 0 || elem_bytes == 0 || (comm->c.rank == 0 && !out_root && n_global > 0)) {
    set_error("atos_comm_gather: invalid argument");
    return ATOS_ERR_INVALID_ARG;
  }
  Comm* c = &comm->c;
  const int P = c->nranks;
  cudaStream_t s = (cudaStream_t)stream;
  DeviceGuard dg(c->device);
  std::vector<int64_t> vb(P), ve(P);
  for (int r = 0; r < P; ++r) atos_partition_range(n_global, P, r, &vb[r], &ve[r]);
  const size_t mine = (size_t)(ve[c->rank] - vb[c->rank]) * elem_bytes;
  if (mine && !slice) {
    set_error("atos_comm_gather: null slice");
    return ATOS_ERR_INVALID_ARG;
  }
  if (c->h_a2a) {
    // host transport: every rank sends its slice to rank 0 only
    std::vector<char> sbuf(std::max<size_t>(mine, 1)), rbuf(c->rank == 0 ? std::max<size_t>(n_global * elem_bytes, 1) : 1);
    if (mine) ATOS_CUDA(cudaMemcpyAsync(sbuf.data(), slice, mine, cudaMemcpyDeviceToHost, s));
    ATOS_CUDA(cudaStreamSynchronize(s));
    std::vector<uint64_t> sb(P, 0), rb(P, 0);
    sb[0] = mine;
    if (c->rank == 0)
      for (int r = 0; r < P; ++r) rb[r] = (uint64_t)(ve[r] - vb[r]) * elem_bytes;
    if (c->h_a2a(c->h_user, sbuf.data(), sb.data(), rbuf.data(), rb.data()) != 0) {
      set_error("atos_comm_gather: host alltoallv failed");
      return ATOS_ERR_NCCL;
    }
    if (c->rank == 0 && n_global) {
      ATOS_CUDA(cudaMemcpyAsync(out_root, rbuf.data(), n_global * elem_bytes, cudaMemcpyHostToDevice, s));
      ATOS_CUDA(cudaStreamSynchronize(s));
    }
    return ATOS_OK;
  }
  NcclApi& api = nccl();
  ncclComm_t nc = (ncclComm_t)c->nccl;
  ATOS_NCCL(api.GroupStart());
  if (c->rank == 0) {
    if (mine) ATOS_CUDA(cudaMemcpyAsync(out_root, slice, mine, cudaMemcpyDeviceToDevice, s));
    for (int r = 1; r < P; ++r) {
      const size_t b = (size_t)(ve[r] - vb[r]) * elem_bytes;
      if (b) ATOS_NCCL(api.Recv((char*)out_root + (size_t)vb[r] * elem_bytes, b, ncclUint8, r, nc, s));
    }
  } else if (mine) {
    ATOS_NCCL(api.Send(slice, mine, ncclUint8, 0, nc, s));
  }
  ATOS_NCCL(api.GroupEnd());
  ATOS_CUDA(cudaStreamSynchronize(s));
  return ATOS_OK;
}

int atos_csr_create_part(atos_csr** out, atos_comm* comm, int64_t n_global, int64_t v_begin, int64_t v_end,
                         int64_t m_local, const int64_t* row_ptr_local, const int32_t* col_global, int where) {
  if (!out || !comm || n_global < 0 || v_begin < 0 || v_end < v_begin || v_end > n_global || m_local < 0 ||
      (v_end > v_begin && !row_ptr_local) || (m_local > 0 && !col_global)) {
    set_error("atos_csr_create_part: invalid argument");
    return ATOS_ERR_INVALID_ARG;
  }
  *out = nullptr;
  int64_t eb = 0, ee = 0;
  atos_partition_range(n_global, comm->c.nranks, comm->c.rank, &eb, &ee);
  if (eb != v_begin || ee != v_end) {
    set_error("atos_csr_create_part: rank %d must own [%lld, %lld) (atos_partition_range), got [%lld, %lld)",
              comm->c.rank, (long long)eb, (long long)ee, (long long)v_begin, (long long)v_end);
    return ATOS_ERR_INVALID_ARG;
  }
  if (m_local >= (int64_t)0xFFFFFFFFll || n_global >= (int64_t)0x7FFFFFFFll) {
    set_error("atos_csr_create_part: n < 2^31 and m_local < 2^32 required");
    return ATOS_ERR_UNSUPPORTED;
  }
  if (where == ATOS_MEM_HOST) {
    const int64_t nl = v_end - v_begin;
    if (nl > 0 && (row_ptr_local[0] != 0 || row_ptr_local[nl] != m_local)) {
      set_error("atos_csr_create_part: row_ptr_local must start at 0 and end at m_local");
      return ATOS_ERR_INVALID_ARG;
    }
    for (int64_t i = 0; i < nl; ++i)
      if (row_ptr_local[i + 1] < row_ptr_local[i]) {
        set_error("atos_csr_create_part: row_ptr_local not non-decreasing at %lld", (long long)i);
        return ATOS_ERR_INVALID_ARG;
      }
    for (int64_t e = 0; e < m_local; ++e)
      if (col_global[e] < 0 || (int64_t)col_global[e] >= n_global) {
        set_error("atos_csr_create_part: col_global[%lld] out of range", (long long)e);
        return ATOS_ERR_INVALID_ARG;
      }
  }
  DeviceGuard dg(comm->c.device);
  atos_csr* g = new atos_csr();
  g->device = comm->c.device;
  g->n = n_global;
  g->m = m_local;
  g->num_parts = 1;
  g->comm = &comm->c;
  g->rank = comm->c.rank;
  g->nranks = comm->c.nranks;
  g->parts.resize(1);
  int rc = upload_part_local(g->parts[0], row_ptr_local, col_global, where, v_end - v_begin, m_local);
  if (rc == ATOS_OK) {
    g->parts[0].v_begin = v_begin;
    g->parts[0].v_end = v_end;
  } else {
    atos_csr_destroy(g);
    return rc;
  }
  *out = g;
  return ATOS_OK;
}

}  // extern "C"
