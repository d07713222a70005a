// Paged KV cache layout (internal).  One page = one (block, kv head): 16 tokens x D bf16, pages
// ordered [kv_blocks][Hkv].  A page is stored "SMEM-ready": D/64 column atoms of [16 rows][64
// elements] (2 KB each), and within a 128-byte atom row the eight 16-byte chunks are XOR-swizzled
// by (row & 7) -- exactly what a 128-byte-swizzle TMA box of 16 x 64 leaves in shared memory.  So a
// page moves with plain copies (one 1-D bulk copy per page in the decode kernel, 16-byte cp.async
// chunks in the prefill kernel) and is read there by ldmatrix / UMMA descriptors as SW128 data:
// 16-row TMA boxes cost ~70 cycles of TMA issue each (tools/micro/tma_box.cu), which capped the
// prefill kernel's K/V stream at ~30 B/cycle per SM.
#pragma once
#include <stdint.h>

namespace gllm {

// element offset of (row, col) inside the cache, page = blk * Hkv + kv_head
__host__ __device__ __forceinline__ int64_t kv_page_elem(int64_t page, int row, int col, int D) {
  const int atom = col >> 6, c16 = (col & 63) >> 3, e = col & 7;
  return page * 16 * D + atom * 1024 + row * 64 + ((c16 ^ (row & 7)) << 3) + e;
}

}  // namespace gllm
