// kernels_p4.cu -- kernel instantiations for table variant VAR_P4 (see kernels_inst.cuh).
#define FSM_VAR speck::VAR_P4
#define FSM_VAR_NAME p4
#include "kernels_inst.cuh"
