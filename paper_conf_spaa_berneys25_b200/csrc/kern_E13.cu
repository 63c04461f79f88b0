// explicit instantiations for E = 13 (see kern_inst.cuh)
#include "kern_inst.cuh"
BCF_DEFINE_REG(13)
