// kernels_common.cuh — device-side includes shared by the kernel units (mat_*.cu).
#pragma once
#include <cuda_bf16.h>
#include <cuda_runtime.h>
#include <stdint.h>

#include "kernels.h"
#include "k_resample.cuh"
#include "k_stream.cuh"
