// kernels_hs.cu -- kernel instantiations for table variant VAR_HS (see kernels_inst.cuh).
#define FSM_VAR speck::VAR_HS
#define FSM_VAR_NAME hs
#include "kernels_inst.cuh"
