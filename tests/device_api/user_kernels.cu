// A USER's CUDA code calling the tilepack device API (include/tilepack/device.cuh): the paper's
// claim that LoadBitPack / LoadDBitPack / LoadRBitPack drop into an ordinary kernel in place of
// a tile load.  Built by __graft_entry__.build() into
// libuser_kernels.so; tests/test_device_api.py checks it against the oracle.  Nothing here
// links libtilepack.so.
#include <cuda_runtime.h>

#include "tilepack/device.cuh"

namespace {

constexpr int BT = 128, ITEMS = 4;  // Crystal's 128 threads x 4 items

template <int SCHEME>
__device__ __forceinline__ void load(const tp_column& c, uint32_t tile, int32_t (&x)[ITEMS], uint32_t* smem) {
  if (SCHEME == TP_FOR) tp_load_for<BT, ITEMS>(c, tile, x, smem);
  else if (SCHEME == TP_DFOR) tp_load_dfor<BT, ITEMS>(c, tile, x, smem);
  else tp_load_rfor<BT, ITEMS>(c, tile, x, smem);
}

// decode a whole column, one tile per block iteration
template <int SCHEME>
__global__ void __launch_bounds__(BT) user_decode(const tp_column c, int32_t* __restrict__ out) {
  __shared__ uint32_t smem[TP_TILE_SMEM_WORDS];
  const uint32_t ntiles = (uint32_t)((c.n + 511u) / 512u);
  for (uint32_t t = blockIdx.x; t < ntiles; t += gridDim.x) {
    int32_t x[ITEMS];
    load<SCHEME>(c, t, x, smem);
    const uint32_t rows = tp_tile_rows(c, t);
#pragma unroll
    for (int k = 0; k < ITEMS; ++k) {
      const uint32_t r = k * BT + threadIdx.x;
      if (r < rows) out[512ull * t + r] = x[k];
    }
  }
}

// SELECT SUM(a * b) WHERE lo <= c <= hi -- a GPU-FOR, b GPU-DFOR, c GPU-RFOR: three decodes
// fused into one query kernel, values in registers
__global__ void __launch_bounds__(BT) user_select_sum(const tp_column a, const tp_column b, const tp_column c,
                                                       int32_t lo, int32_t hi, unsigned long long* out) {
  __shared__ uint32_t smem[TP_TILE_SMEM_WORDS];
  const uint32_t ntiles = (uint32_t)((a.n + 511u) / 512u);
  long long acc = 0;
  for (uint32_t t = blockIdx.x; t < ntiles; t += gridDim.x) {
    int32_t xa[ITEMS], xb[ITEMS], xc[ITEMS];
    tp_load_rfor<BT, ITEMS>(c, t, xc, smem);
    tp_load_for<BT, ITEMS>(a, t, xa, smem);
    tp_load_dfor<BT, ITEMS>(b, t, xb, smem);
    const uint32_t rows = tp_tile_rows(a, t);
#pragma unroll
    for (int k = 0; k < ITEMS; ++k) {
      const uint32_t r = k * BT + threadIdx.x;
      if (r < rows && xc[k] >= lo && xc[k] <= hi) acc += (long long)xa[k] * xb[k];
    }
  }
  for (int d = 16; d > 0; d >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, d);
  if ((threadIdx.x & 31u) == 0) atomicAdd(out, (unsigned long long)acc);
}

}  // namespace

extern "C" {

int user_decode_launch(const tp_column* c, int32_t* d_out, void* stream) {
  const int grid = 148 * 8;
  auto s = (cudaStream_t)stream;
  if (c->scheme == TP_FOR) user_decode<TP_FOR><<<grid, BT, 0, s>>>(*c, d_out);
  else if (c->scheme == TP_DFOR) user_decode<TP_DFOR><<<grid, BT, 0, s>>>(*c, d_out);
  else if (c->scheme == TP_RFOR) user_decode<TP_RFOR><<<grid, BT, 0, s>>>(*c, d_out);
  else return 1;
  return cudaGetLastError() == cudaSuccess ? 0 : 4;
}

int user_select_sum_launch(const tp_column* a, const tp_column* b, const tp_column* c, int32_t lo, int32_t hi,
                           int64_t* d_out, void* stream) {
  if (a->scheme != TP_FOR || b->scheme != TP_DFOR || c->scheme != TP_RFOR) return 1;
  user_select_sum<<<148 * 8, BT, 0, (cudaStream_t)stream>>>(*a, *b, *c, lo, hi,
                                                           reinterpret_cast<unsigned long long*>(d_out));
  return cudaGetLastError() == cudaSuccess ? 0 : 4;
}

}  // extern "C"
