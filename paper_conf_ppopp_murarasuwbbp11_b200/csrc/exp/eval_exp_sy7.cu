// SY7: CTA barrier at every level step of dimension 7
#include "exp_sync.cuh"
SG_SYNC(exp_SY7, 7)
