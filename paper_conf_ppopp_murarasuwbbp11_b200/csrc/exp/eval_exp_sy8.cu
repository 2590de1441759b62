// SY8: CTA barrier at every level step of dimension 8
#include "exp_sync.cuh"
SG_SYNC(exp_SY8, 8)
