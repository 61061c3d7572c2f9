// spmv_ws.cuh -- warp-specialised slate worker of the CSR SpMV kind; see spmv_ws.cu.
#pragma once
#include "kernels.h"
namespace slate {
KindOps spmv_ws_ops();
}
