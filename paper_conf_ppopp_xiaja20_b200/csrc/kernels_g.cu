// kernels_g.cu -- kernel instantiations for table variant VAR_G (see kernels_inst.cuh).
#define FSM_VAR speck::VAR_G
#define FSM_VAR_NAME g
#include "kernels_inst.cuh"
