// SY9: CTA barrier at every level step of dimension 9
#include "exp_sync.cuh"
SG_SYNC(exp_SY9, 9)
