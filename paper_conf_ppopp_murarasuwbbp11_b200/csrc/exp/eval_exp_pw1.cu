// PW1: the v9 product launch structure with persistent SM-affine warps (exp_pw.cuh)
#include "exp_v9.cuh"
SG_V9(exp_PW1, true, false, false, 256, 2, 128, 3, true)
