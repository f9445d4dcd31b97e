// ntt_tensor.cuh -- tcgen05 int8 tensor-core path.  [stub: filled in next]
#pragma once
#include <cstdint>
#include <vector>
#include "ntt_cuda_core.cuh"

namespace wd {

struct TensorTables {
    void* d_planes = nullptr;
};

inline bool tensor_supported(uint32_t) { return false; }
inline float default_tensor_share(uint32_t) { return 0.0f; }
inline int build_tensor_tables(TensorTables&, uint32_t, const std::vector<uint32_t>&, const std::vector<uint32_t>&) { return 0; }
inline void free_tensor_tables(TensorTables& t) { if (t.d_planes) cudaFree(t.d_planes); t.d_planes = nullptr; }
inline int prepare_tensor_kernels(uint32_t) { return 0; }
inline int launch_tensor(uint32_t, bool, const NttArgs&, const TensorTables&, uint32_t, float, cudaStream_t) { return -1; }

}  // namespace wd
