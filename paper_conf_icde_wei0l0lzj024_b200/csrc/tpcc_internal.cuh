// TPC-C PROC-mode scratch and launchers (stored procedures).
#pragma once
#include "ltpg_internal.cuh"

namespace ltpg {

struct TpccDev {
  uint32_t max_txns = 0;
  int* by_name = nullptr;  // dense secondary index [(w*10+d)*1000 + last] -> c_id
  uint32_t n_by_name = 0;
};

int tpcc_alloc(TpccDev& t, uint32_t max_txns);
void tpcc_free(TpccDev& t);
int tpcc_build_secondary(TpccDev& t, const DevTable* h_tab, const DevTable* d_tab, uint32_t n_warehouses);
int tpcc_run(TpccDev& t, const DevTable* h_tab, const DevTable* d_tab, BatchDev& b, const ltpg_config& cfg,
             cudaStream_t s, cudaEvent_t* ev);

}  // namespace ltpg
