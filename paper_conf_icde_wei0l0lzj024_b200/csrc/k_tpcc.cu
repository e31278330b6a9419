// TPC-C PROC mode (placeholder until the procedure kernels land).
#include "tpcc_internal.cuh"

namespace ltpg {
LTPG_DEFINE_TABLE_UPLOAD(upload_tables_tpcc)
int tpcc_alloc(TpccDev& t, uint32_t max_txns) { t.max_txns = max_txns; return 0; }
void tpcc_free(TpccDev& t) { (void)t; }
int tpcc_build_secondary(TpccDev&, const DevTable*, const DevTable*, uint32_t) { return 0; }
int tpcc_run(TpccDev&, const DevTable*, const DevTable*, BatchDev&, const ltpg_config&, cudaStream_t, cudaEvent_t*) {
  return LTPG_EINVAL;
}
}  // namespace ltpg
