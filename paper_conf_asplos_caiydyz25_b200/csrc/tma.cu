// Host-side tensor maps for the TMA loads of libsmoothe (sm_100a).  Encoded
// through the driver entry point (the library links the static runtime only)
// and cached per (pointer, shape, box): kernels take them by value as
// __grid_constant__ parameters, so a captured CUDA graph keeps its copy.
#include <cuda.h>

#include <mutex>
#include <vector>

#include "internal.h"

namespace smoothe {

// Returned by value: the cache is a growing vector, so a reference into it
// would dangle as soon as a later call adds an entry (a second map encoded
// for the same launch corrupted the first one's copy: illegal instruction).
CUtensorMap tensor_map_2d(const void* base, bool is_int, uint64_t inner, uint64_t outer,
                          uint64_t row_bytes, uint32_t box_inner, uint32_t box_outer,
                          bool swizzle128) {
  struct Entry {
    const void* p;
    bool i;
    uint64_t in, out, rb;
    uint32_t bi, bo;
    bool sw;
    CUtensorMap m;
  };
  typedef CUresult (*EncodeFn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*,
                               const cuuint64_t*, const cuuint64_t*, const cuuint32_t*,
                               const cuuint32_t*, CUtensorMapInterleave, CUtensorMapSwizzle,
                               CUtensorMapL2promotion, CUtensorMapFloatOOBfill);
  static std::mutex mu;
  static std::vector<Entry> cache;
  static EncodeFn encode = nullptr;
  std::lock_guard<std::mutex> lk(mu);
  for (auto& e : cache)
    if (e.p == base && e.i == is_int && e.in == inner && e.out == outer && e.rb == row_bytes &&
        e.bi == box_inner && e.bo == box_outer && e.sw == swizzle128)
      return e.m;
  if (!encode) {
    void* fn = nullptr;
    cudaDriverEntryPointQueryResult q;
    SM_CUDA(cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fn, cudaEnableDefault, &q));
    SM_REQUIRE(fn && q == cudaDriverEntryPointSuccess, SMOOTHE_E_CUDA,
               "cuTensorMapEncodeTiled unavailable");
    encode = (EncodeFn)fn;
  }
  Entry e{base, is_int, inner, outer, row_bytes, box_inner, box_outer, swizzle128, {}};
  const cuuint64_t dims[2] = {inner, outer};
  const cuuint64_t strides[1] = {row_bytes};
  const cuuint32_t box[2] = {box_inner, box_outer}, es[2] = {1, 1};
  const CUresult r = encode(&e.m, is_int ? CU_TENSOR_MAP_DATA_TYPE_INT32 : CU_TENSOR_MAP_DATA_TYPE_FLOAT32,
                            2, const_cast<void*>(base), dims, strides, box, es,
                            CU_TENSOR_MAP_INTERLEAVE_NONE,
                            swizzle128 ? CU_TENSOR_MAP_SWIZZLE_128B : CU_TENSOR_MAP_SWIZZLE_NONE,
                            CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  SM_REQUIRE(r == CUDA_SUCCESS, SMOOTHE_E_CUDA, "cuTensorMapEncodeTiled failed");
  if (cache.size() > 512) cache.erase(cache.begin());
  cache.push_back(e);
  return cache.back().m;
}

}  // namespace smoothe
