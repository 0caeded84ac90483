// Instantiation of the generic evaluator (dag_eval.cuh) for K = 4 samples
// per thread (joint / marginal x shared-memory / global feature source).
#include "dag_eval.cuh"
namespace spnb {
SPNB_INSTANTIATE_K(4)
}  // namespace spnb
