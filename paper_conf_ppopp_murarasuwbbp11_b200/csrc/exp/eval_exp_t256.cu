// T256: r02 v9 experiment variant (exp_v9.cuh)
#include "exp_v9.cuh"
SG_V9(exp_T256, false, false, false, 256, 2, 128, 3)
