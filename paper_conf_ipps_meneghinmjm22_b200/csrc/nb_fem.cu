// nb_fem.cu — matrix-free Q1 linear-elastic operator.
// Placeholder: the FEM 27-point row (a10) is built after a1-a9.
#include "nb_internal.cuh"

nb_status nb_fem_cg_hooks(nb_cg *, int) { NB_FAIL(NB_EUNSUPPORTED, "FEM operator not built yet"); }
nb_status nb_fem_cg_init(nb_cg *) { NB_FAIL(NB_EUNSUPPORTED, "FEM operator not built yet"); }
extern "C" nb_status nb_fem27_apply(const nb_field *, nb_field *, double, double) {
    NB_FAIL(NB_EUNSUPPORTED, "FEM operator not built yet");
}
extern "C" nb_status nb_fem27_rhs(nb_field *, double) { NB_FAIL(NB_EUNSUPPORTED, "FEM operator not built yet"); }
