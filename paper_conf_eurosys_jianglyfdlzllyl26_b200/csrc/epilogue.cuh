// Fused GEMM epilogue (bias, GELU, gated residual, row-scatter routing) -- see Epilogue in
// common.cuh.  PAPER.md L146/L157: the QKV epilogue scatters fresh K/V rows into the merged key
// buffer at their original token rows, so attention sees fresh + cached keys in token order.
#pragma once
#include "common.cuh"

namespace fps {

// Apply the epilogue to NC consecutive columns c0..c0+NC-1 of row r (NC | 8, c0 % NC == 0,
// and all NC columns on the same side of `split`, `split2` and `act_from`).  Vectorised 16-B stores when possible.
template <typename T, int NC>
__device__ __forceinline__ void epilogue_store(const Epilogue& ep, int r, int c0, float* v) {
  if (ep.bias) {
    const T* b = reinterpret_cast<const T*>(ep.bias) + c0;
#pragma unroll
    for (int e = 0; e < NC; ++e) v[e] += to_f(b[e]);
  }
  if (ep.act == 1 && c0 >= ep.act_from) {
#pragma unroll
    for (int e = 0; e < NC; ++e) v[e] = gelu_tanh(v[e]);
  }
  if (ep.resid) {
    const int rr = ep.resid_map ? __ldg(ep.resid_map + r) : r;
    const T* res = reinterpret_cast<const T*>(ep.resid) + (size_t)rr * ep.ld_resid + c0;
    if (ep.gate) {
      const int q = find_req(ep.cu, ep.n_req, r);
      const T* g = reinterpret_cast<const T*>(ep.gate) + (size_t)q * ep.gate_stride + c0;
#pragma unroll
      for (int e = 0; e < NC; ++e) v[e] = to_f(res[e]) + to_f(g[e]) * v[e];
    } else {
#pragma unroll
      for (int e = 0; e < NC; ++e) v[e] = to_f(res[e]) + v[e];
    }
  }
  T* dst;
  if (c0 < ep.split) {
    const int orow = ep.map0 ? __ldg(ep.map0 + r) : r;
    dst = reinterpret_cast<T*>(ep.out0) + (size_t)orow * ep.ld0 + c0;
  } else if (ep.out2 && c0 >= ep.split2) {
    dst = reinterpret_cast<T*>(ep.out2) + (size_t)r * ep.ld2 + (c0 - ep.split2);
  } else {
    const int orow = ep.map1 ? __ldg(ep.map1 + r) : r;
    dst = reinterpret_cast<T*>(ep.out1) + (size_t)orow * ep.ld1 + (c0 - ep.split);
  }
  if constexpr (NC * sizeof(T) == 16) {
    *reinterpret_cast<uint4*>(dst) = Vec16<T>::pack(v);
  } else {
#pragma unroll
    for (int e = 0; e < NC; ++e) dst[e] = from_f<T>(v[e]);
  }
}

}  // namespace fps
