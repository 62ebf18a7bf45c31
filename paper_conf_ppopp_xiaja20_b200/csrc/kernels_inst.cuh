// kernels_inst.cuh -- explicit instantiation of every kernel for one table variant.  Included by
// kernels_<variant>.cu with FSM_VAR / FSM_VAR_NAME defined; the host (fsmspec.cu) reaches the
// kernels through the accessors defined here.  K list = kKs in fsmspec.cu.
#include "fixup_kernel.cuh"
#include "seqmerge_kernel.cuh"
#include "spec_kernel.cuh"
#include "speck_kernel.cuh"

using namespace speck;
typedef void (*KernelFn)(Params);
typedef void (*FixFn)(FixParams);
typedef void (*SeqLocalFn)(Params, SeqBuf);
typedef void (*SeqWalkFn)(Params, SeqBuf);
typedef void (*SpecFn)(Params, uint16_t *);
typedef void (*MultiFn)(Params, const Params *, uint32_t);

#define FSM_CAT2(a, b) a##b
#define FSM_CAT(a, b) FSM_CAT2(a, b)

// Alg. 2 (hash check) kernels exist for the large-k instantiations only (the paper uses the hash
// form for k > 12); the host falls back to Alg. 1 elsewhere.
template <int K>
static KernelFn pick(bool split, bool hash)
{
    if constexpr (K >= 12) {
        if (hash) return speck_kernel<K, FSM_VAR, false, true>;  // Alg. 2 kernels are unsplit
    }
    if constexpr (split_kernel(FSM_VAR, K)) {
        if (split) return speck_kernel<K, FSM_VAR, true>;
    }
    return speck_kernel<K, FSM_VAR, false>;
}

KernelFn FSM_CAT(get_kernel_, FSM_VAR_NAME)(int K, bool split, bool hash)
{
    switch (K) {
    case 1: return pick<1>(split, false);
    case 2: return pick<2>(split, false);
    case 3: return pick<3>(split, false);
    case 4: return pick<4>(split, false);
    case 6: return pick<6>(split, false);
    case 8: return pick<8>(split, false);
    case 12: return pick<12>(split, hash);
    default: return pick<16>(split, hash);
    }
}

MultiFn FSM_CAT(get_multi_, FSM_VAR_NAME)(int K)
{
    switch (K) {
    case 1: return speck_multi_kernel<1, FSM_VAR>;
    case 2: return speck_multi_kernel<2, FSM_VAR>;
    case 3: return speck_multi_kernel<3, FSM_VAR>;
    case 4: return speck_multi_kernel<4, FSM_VAR>;
    case 6: return speck_multi_kernel<6, FSM_VAR>;
    case 8: return speck_multi_kernel<8, FSM_VAR>;
    default: return nullptr;  // K >= 12: the host runs those DFAs one launch each
    }
}

FixFn FSM_CAT(get_fix_, FSM_VAR_NAME)() { return fixup_kernel<FSM_VAR>; }

void FSM_CAT(get_seq_, FSM_VAR_NAME)(int K, SeqLocalFn &l, SeqWalkFn &w)
{
    switch (K) {
    case 1: l = seq_local_kernel<1, FSM_VAR>; w = seq_walk_kernel<1, FSM_VAR>; break;
    case 2: l = seq_local_kernel<2, FSM_VAR>; w = seq_walk_kernel<2, FSM_VAR>; break;
    case 3: l = seq_local_kernel<3, FSM_VAR>; w = seq_walk_kernel<3, FSM_VAR>; break;
    case 4: l = seq_local_kernel<4, FSM_VAR>; w = seq_walk_kernel<4, FSM_VAR>; break;
    case 6: l = seq_local_kernel<6, FSM_VAR>; w = seq_walk_kernel<6, FSM_VAR>; break;
    case 8: l = seq_local_kernel<8, FSM_VAR>; w = seq_walk_kernel<8, FSM_VAR>; break;
    case 12: l = seq_local_kernel<12, FSM_VAR>; w = seq_walk_kernel<12, FSM_VAR>; break;
    default: l = seq_local_kernel<16, FSM_VAR>; w = seq_walk_kernel<16, FSM_VAR>; break;
    }
}

SpecFn FSM_CAT(get_spec_, FSM_VAR_NAME)() { return spec_kernel<FSM_VAR>; }
