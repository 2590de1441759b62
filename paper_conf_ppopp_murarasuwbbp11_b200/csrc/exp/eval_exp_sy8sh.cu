// SY8S / SY8H: the dimension-8 barrier only in the small-block / only in the large-block launches
#include "exp_sync.cuh"
SG_SYNC2(exp_SY8S, 8, -1)
SG_SYNC2(exp_SY8H, -1, 8)
