// kernels_h8.cu -- kernel instantiations for table variant VAR_H8 (see kernels_inst.cuh).
#define FSM_VAR speck::VAR_H8
#define FSM_VAR_NAME h8
#include "kernels_inst.cuh"
