// kernels_r16.cu -- kernel instantiations for table variant VAR_R16 (see kernels_inst.cuh).
#define FSM_VAR speck::VAR_R16
#define FSM_VAR_NAME r16
#include "kernels_inst.cuh"
