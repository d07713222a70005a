// Varlen paged causal attention over one mixed batch (a7 of DESIGN.md §2) -- internal interface.
#pragma once
#include <cuda.h>
#include <cuda_bf16.h>
#include <cuda_runtime.h>
#include <stdint.h>

namespace gllm {

// work item of the prefill kernel: chunk `seq`, flattened (token, group-head) rows [row0, row0+rows_per_item)
struct PrefillItem {
  int32_t seq, row0;
};
// work item of the decode kernel: decode row `seq`, key split `split`; `part` = partial slot or -1
struct DecodeItem {
  int32_t seq, split, part, nsplit;
};
// merge job: decode seq `seq`, partial slots [first, first + nsplit)
struct MergeItem {
  int32_t seq, first, nsplit, pad;
};

struct AttnArgs {
  const __nv_bfloat16* q;  // [T, q_stride] (rotated q heads first in each row)
  int q_stride;
  const __nv_bfloat16* kc;  // [kv_blocks][Hkv] pages of bs x D, SMEM-ready layout (kvpage.cuh)
  const __nv_bfloat16* vc;
  int Hq, Hkv, D, bs;
  const int32_t* cu_q;
  const int32_t* kv_len;
  const int32_t* block_table;
  int maxblk;
  __nv_bfloat16* out;  // [T, Hq*D]
  float* part_o;       // [nparts, Hkv, G, D]
  float* part_ml;      // [nparts, Hkv, G, 2]
  int split_len;       // decode keys per split (multiple of 16)
  int* part_ctr;       // [nparts * Hkv] split arrival counters (persistent decode kernel; kept zero)
};

// warp-specialised tcgen05 prefill (attention_prefill_ws.cu): items of prefill_ws_rows_per_item()
// rows (two 128-row Q tiles); K / V pages (SMEM-ready layout, kvpage.cuh) by 16-byte cp.async
int prefill_ws_rows_per_item();
int launch_prefill_attention_ws(const AttnArgs& a, const PrefillItem* items, int n_items, cudaStream_t s);
// persistent warp-worker decode kernel (attention_decode.cu): each K / V page (SMEM-ready layout,
// kvpage.cuh) is one 1-D bulk copy; `ctr` = 2 device ints, zero before the first launch (the kernel
// leaves them zero)
bool decode_tma_supported(int D, int G);
int decode_workers(int num_sms);  // warp workers of the persistent decode kernel
int launch_decode_attention_tma(const AttnArgs& a, const DecodeItem* items, int n_items, const MergeItem* merges,
                                int n_merges, int* ctr, int num_sms, cudaStream_t s);

}  // namespace gllm
