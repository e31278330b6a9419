// a9 host retry loop: compose the next batch from the
// previous batch's conflict aborts (original TIDs, ascending ranks) and a prefix of fresh txns.
// Host-side copies only; no db, no device.
#include <cstring>

#include "ltpg_internal.cuh"

namespace {

// txns [begin, end) of an OPS batch, op range of txn r
inline uint32_t ops_of(const ltpg_batch* b, uint32_t r) { return b->op_begin[r + 1] - b->op_begin[r]; }

}  // namespace

extern "C" int ltpg_compose_retry(const ltpg_batch* prev, const uint32_t* abort_idx, uint32_t n_aborted,
                                  const ltpg_batch* fresh, ltpg_batch_buf* out) {
  if (!prev || !fresh || !out || (n_aborted && !abort_idx) || !out->tid) return LTPG_EINVAL;
  if (prev->mode != fresh->mode || prev->inputs_on_device || fresh->inputs_on_device) return LTPG_EINVAL;
  if ((prev->n_txns && !prev->tid) || (fresh->n_txns && !fresh->tid)) return LTPG_EINVAL;
  const bool ops = prev->mode == LTPG_MODE_OPS;
  if (!ops && prev->mode != LTPG_MODE_TPCC) return LTPG_EINVAL;
  if (ops) {
    if (!out->op_begin || (out->cap_ops && (!out->ops || !out->op_arg))) return LTPG_EINVAL;
    if ((prev->n_txns && !prev->op_begin) || (fresh->n_txns && !fresh->op_begin)) return LTPG_EINVAL;
    if ((prev->n_ops && (!prev->ops || !prev->op_arg)) || (fresh->n_ops && (!fresh->ops || !fresh->op_arg)))
      return LTPG_EINVAL;
  } else {
    if (prev->proc_offsets || fresh->proc_offsets) return LTPG_EINVAL;  // packed blocks: not here
    if ((prev->n_txns && (!prev->proc_type || !prev->proc_params)) ||
        (fresh->n_txns && (!fresh->proc_type || !fresh->proc_params)))
      return LTPG_EINVAL;
    if ((out->cap_txns && (!out->proc_type || !out->proc_params))) return LTPG_EINVAL;
  }
  if (n_aborted > out->cap_txns) return LTPG_EINVAL;
  // validate the abort list and count the retried ops before writing anything
  uint64_t retried_ops = 0;
  for (uint32_t i = 0; i < n_aborted; ++i) {
    const uint32_t r = abort_idx[i];
    if (r >= prev->n_txns || (i && r <= abort_idx[i - 1])) return LTPG_EINVAL;
    if (ops) retried_ops += ops_of(prev, r);
  }
  if (ops && retried_ops > out->cap_ops) return LTPG_EINVAL;
  const uint64_t last_tid = n_aborted ? prev->tid[abort_idx[n_aborted - 1]] : 0;
  if (n_aborted && fresh->n_txns && fresh->tid[0] <= last_tid) return LTPG_EINVAL;
  // fresh prefix that fits
  uint32_t nf = 0;
  uint64_t fresh_ops = 0;
  while (nf < fresh->n_txns && n_aborted + nf < out->cap_txns) {
    if (ops) {
      const uint32_t k = ops_of(fresh, nf);
      if (retried_ops + fresh_ops + k > out->cap_ops) break;
      fresh_ops += k;
    }
    ++nf;
  }
  // retried txns, in rank order, then the fresh prefix
  uint32_t n = 0, m = 0;
  if (ops) out->op_begin[0] = 0;
  for (uint32_t i = 0; i < n_aborted; ++i, ++n) {
    const uint32_t r = abort_idx[i];
    out->tid[n] = prev->tid[r];
    if (ops) {
      const uint32_t b0 = prev->op_begin[r], k = ops_of(prev, r);
      std::memcpy(out->ops + m, prev->ops + b0, k * sizeof(ltpg_op));
      std::memcpy(out->op_arg + m, prev->op_arg + b0, k * sizeof(int64_t));
      m += k;
      out->op_begin[n + 1] = m;
    } else {
      out->proc_type[n] = prev->proc_type[r];
      std::memcpy(out->proc_params + (size_t)n * LTPG_PARAM_BYTES, prev->proc_params + (size_t)r * LTPG_PARAM_BYTES,
                  LTPG_PARAM_BYTES);
    }
  }
  if (nf) {
    std::memcpy(out->tid + n, fresh->tid, nf * sizeof(uint64_t));
    if (ops) {
      const uint32_t f0 = fresh->op_begin[0], k = (uint32_t)fresh_ops;
      std::memcpy(out->ops + m, fresh->ops + f0, k * sizeof(ltpg_op));
      std::memcpy(out->op_arg + m, fresh->op_arg + f0, k * sizeof(int64_t));
      for (uint32_t j = 0; j < nf; ++j) out->op_begin[n + j + 1] = m + (fresh->op_begin[j + 1] - f0);
      m += k;
    } else {
      std::memcpy(out->proc_type + n, fresh->proc_type, nf);
      std::memcpy(out->proc_params + (size_t)n * LTPG_PARAM_BYTES, fresh->proc_params, (size_t)nf * LTPG_PARAM_BYTES);
    }
    n += nf;
  }
  out->n_txns = n;
  out->n_ops = m;
  out->n_retried = n_aborted;
  out->n_fresh = nf;
  return LTPG_OK;
}

// SURVEY §8(e) routing: the shard of `rank` (txns touching its warehouses, in order, with their
// global ranks).  Host-side copies only; part_of_w is the device's ownership rule.
extern "C" int ltpg_route_tpcc(const ltpg_batch* g, uint32_t nw, uint32_t world, uint32_t rank, ltpg_batch_buf* out,
                               uint32_t* grank) {
  if (!g || !out || !grank || g->mode != LTPG_MODE_TPCC || g->inputs_on_device || g->proc_offsets || !world ||
      rank >= world || !nw || (g->n_txns && (!g->tid || !g->proc_type || !g->proc_params)) || !out->tid ||
      (out->cap_txns && (!out->proc_type || !out->proc_params)))
    return LTPG_EINVAL;
  auto part = [&](uint32_t w) { return ltpg::part_of_w(w, nw, world); };
  uint32_t n = 0;
  for (uint32_t r = 0; r < g->n_txns; ++r) {
    const uint8_t* p = g->proc_params + (size_t)r * LTPG_PARAM_BYTES;
    const uint32_t w = p[0] | (uint32_t)p[1] << 8;
    bool mine = part(w) == rank;
    if (!mine && g->proc_type[r] == LTPG_NEW_ORDER)
      for (uint32_t l = 0; l < p[3] && l < 15 && !mine; ++l) {
        const uint8_t* L = p + 8 + 8 * l;
        mine = part(L[4] | (uint32_t)L[5] << 8) == rank;
      }
    if (!mine && g->proc_type[r] == LTPG_PAYMENT) mine = part(p[4] | (uint32_t)p[5] << 8) == rank;
    if (!mine) continue;
    if (n >= out->cap_txns) return LTPG_EINVAL;
    out->tid[n] = g->tid[r];
    out->proc_type[n] = g->proc_type[r];
    std::memcpy(out->proc_params + (size_t)n * LTPG_PARAM_BYTES, p, LTPG_PARAM_BYTES);
    grank[n] = r;
    ++n;
  }
  out->n_txns = n;
  out->n_ops = 0;
  out->n_retried = 0;
  out->n_fresh = n;
  return LTPG_OK;
}
