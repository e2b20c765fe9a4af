// inst_f64.cu -- the driver and kernels instantiated for double.
#define SS_INST_T double
#include "driver.cuh"
