// gemm_tc.cuh -- tensor-core bf16 GEMM tenant (tcgen05 + TMA + TMEM); see gemm_tc.cu.
#pragma once
#include "kernels.h"
namespace slate {
KindOps gemm_tc_ops();
}
