// kernels_b.cu -- kernel instantiations for table variant VAR_B (see kernels_inst.cuh).
#define FSM_VAR speck::VAR_B
#define FSM_VAR_NAME b
#include "kernels_inst.cuh"
