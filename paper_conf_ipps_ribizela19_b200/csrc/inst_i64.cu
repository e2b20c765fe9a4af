// inst_i64.cu -- the driver and kernels instantiated for long long.
#define SS_INST_T long long
#include "driver.cuh"
