// kernels_cl.cu -- kernel instantiations for table variant VAR_CL (see kernels_inst.cuh).
#define FSM_VAR speck::VAR_CL
#define FSM_VAR_NAME cl
#include "kernels_inst.cuh"
