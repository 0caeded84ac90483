// Instantiation of the generic evaluator (dag_eval.cuh) for K = 8 samples
// per thread (register stack depth 10; joint / marginal x feature source).
#include "dag_eval.cuh"
namespace spnb {
SPNB_INSTANTIATE_K(8)
}  // namespace spnb
