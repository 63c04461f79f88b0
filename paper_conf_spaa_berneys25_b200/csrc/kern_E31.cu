// explicit instantiations for E = 31 (see kern_inst.cuh)
#include "kern_inst.cuh"
BCF_DEFINE_REG(31)
