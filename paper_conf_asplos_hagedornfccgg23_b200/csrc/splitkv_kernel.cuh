// splitkv_kernel.cuh — the merge step of split-KV FMHA (fmha_fwd_splitkv).
//
// The FMHA kernel in MODE_SPLIT computes, for split s of a row's keys (KV tiles
// [s * split_tiles, (s + 1) * split_tiles)), the online-softmax state of PAPER.md L487's softmax
// restricted to those keys: an exp2 reference mc_s (= scale * log2 e * a running max), the row sum
// l_s = sum_j 2^(c S_ij - mc_s) and the unnormalised O_s = sum_j 2^(c S_ij - mc_s) V_j.  The full
// softmax row is their rescaled sum:
//     M = max_s mc_s,   O = sum_s 2^(mc_s - M) O_s / sum_s 2^(mc_s - M) l_s
// (rows with no visible key: l = 0 everywhere -> O = 0, R4).  HBM-bound: one warp per
// output row, each lane D / 32 contiguous elements; fp32 throughout, one RNE rounding at the end.
#pragma once
#include "sm100.cuh"

namespace b200 {

template <int D, bool BF16>
__global__ void __launch_bounds__(256) fmha_splitkv_combine_kernel(const float* __restrict__ ws_o,
                                                                   const float* __restrict__ ws_m,
                                                                   const float* __restrict__ ws_l, void* O,
                                                                   int splits, long long rows) {
  const long long row = (static_cast<long long>(blockIdx.x) * blockDim.x + threadIdx.x) >> 5;
  if (row >= rows) return;
  const int lane = threadIdx.x & 31;
  constexpr int E = D / 32;  // 2 (D = 64) or 4 (D = 128) elements per lane
  float mx = -INFINITY;
  for (int s = 0; s < splits; ++s) mx = fmaxf(mx, __ldg(ws_m + s * rows + row));
  float acc[E];
#pragma unroll
  for (int e = 0; e < E; ++e) acc[e] = 0.f;
  float lsum = 0.f;
  if (mx != -INFINITY) {
    for (int s = 0; s < splits; ++s) {
      const float m = __ldg(ws_m + s * rows + row);
      if (m == -INFINITY) continue;  // no visible key in this split
      const float wgt = exp2f(m - mx);
      lsum += wgt * __ldg(ws_l + s * rows + row);
      const float* src = ws_o + (s * rows + row) * D + lane * E;
      if constexpr (E == 2) {
        const float2 v = __ldg(reinterpret_cast<const float2*>(src));
        acc[0] += wgt * v.x;
        acc[1] += wgt * v.y;
      } else {
        const float4 v = __ldg(reinterpret_cast<const float4*>(src));
        acc[0] += wgt * v.x;
        acc[1] += wgt * v.y;
        acc[2] += wgt * v.z;
        acc[3] += wgt * v.w;
      }
    }
  }
  const float inv = lsum > 0.f ? 1.f / lsum : 0.f;
  uint32_t out[E / 2];
#pragma unroll
  for (int e = 0; e < E / 2; ++e) out[e] = pack2<BF16>(acc[2 * e] * inv, acc[2 * e + 1] * inv);
  uint8_t* dst = static_cast<uint8_t*>(O) + (row * D + lane * E) * 2;
  if constexpr (E == 2)
    *reinterpret_cast<uint32_t*>(dst) = out[0];
  else
    *reinterpret_cast<uint2*>(dst) = make_uint2(out[0], out[1]);
}

}  // namespace b200
