// T256L1: r02 v9 experiment variant (exp_v9.cuh)
#include "exp_v9.cuh"
SG_V9(exp_T256L1, false, false, false, 256, 2, 384, 1)
