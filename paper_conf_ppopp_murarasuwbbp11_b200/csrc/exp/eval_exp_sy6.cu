// SY6: CTA barrier at every level step of dimension 6
#include "exp_sync.cuh"
SG_SYNC(exp_SY6, 6)
