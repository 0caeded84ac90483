// Instantiation of the generic evaluator (dag_eval.cuh) for K = 2 samples
// per thread (joint / marginal x shared-memory / global feature source).
#include "dag_eval.cuh"
namespace spnb {
SPNB_INSTANTIATE_K(2)
}  // namespace spnb
