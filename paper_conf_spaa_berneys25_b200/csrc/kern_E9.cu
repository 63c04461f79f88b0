// explicit instantiations for E = 9 (see kern_inst.cuh)
#include "kern_inst.cuh"
BCF_DEFINE_REG(9)
