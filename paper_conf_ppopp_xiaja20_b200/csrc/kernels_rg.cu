// kernels_rg.cu -- kernel instantiations for table variant VAR_RG (see kernels_inst.cuh).
#define FSM_VAR speck::VAR_RG
#define FSM_VAR_NAME rg
#include "kernels_inst.cuh"
