// dist.cu -- partitioned BFS / PageRank (loopback partitions on one device,
// or one partition per process over NCCL).  Filled in below.
#include "internal.h"

namespace atos {

int create_loopback_parts(atos_csr* g, const int64_t* row_ptr, const int32_t* col, int where) {
  set_error("partitioned graphs not built yet");
  return ATOS_ERR_UNSUPPORTED;
}
int bfs_partitioned(atos_csr* g, int64_t src, uint32_t* depth_dev, const Resolved& r, atos_stats* st) {
  set_error("partitioned BFS not built yet");
  return ATOS_ERR_UNSUPPORTED;
}
int pagerank_partitioned(atos_csr* g, double alpha, double eps, double* rank_dev, const Resolved& r,
                         atos_stats* st) {
  set_error("partitioned PageRank not built yet");
  return ATOS_ERR_UNSUPPORTED;
}

}  // namespace atos

extern "C" {
int atos_comm_unique_id(void* id_out, size_t len) {
  atos::set_error("NCCL communicator not built yet");
  return ATOS_ERR_UNSUPPORTED;
}
int atos_comm_create(atos_comm** out, int nranks, int rank, const void* id, size_t len, int device) {
  atos::set_error("NCCL communicator not built yet");
  return ATOS_ERR_UNSUPPORTED;
}
void atos_comm_destroy(atos_comm* comm) {}
int atos_csr_create_part(atos_csr** out, atos_comm* comm, int64_t n_global, int64_t v_begin, int64_t v_end,
                         int64_t m_local, const int64_t* row_ptr_local, const int32_t* col_global, int where) {
  atos::set_error("partitioned graphs not built yet");
  return ATOS_ERR_UNSUPPORTED;
}
}
