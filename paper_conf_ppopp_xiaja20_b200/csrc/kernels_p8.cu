// kernels_p8.cu -- kernel instantiations for table variant VAR_P8 (see kernels_inst.cuh).
#define FSM_VAR speck::VAR_P8
#define FSM_VAR_NAME p8
#include "kernels_inst.cuh"
