// kernels_n8.cu -- kernel instantiations for table variant VAR_N8 (see kernels_inst.cuh).
#define FSM_VAR speck::VAR_N8
#define FSM_VAR_NAME n8
#include "kernels_inst.cuh"
