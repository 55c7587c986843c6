// nb_sparse.cu — element-sparse grid.  Placeholder:
// the element-sparse grid is the next §8 row (a9) to build.
#include "nb_internal.cuh"

void nb_sparse_free(nb_grid *g) { (void)g; }
nb_status nb_sparse_field_alloc(nb_field *) { NB_FAIL(NB_EUNSUPPORTED, "element-sparse grid not built yet"); }
nb_status nb_sparse_upload(nb_field *, const void *) { NB_FAIL(NB_EUNSUPPORTED, "sparse"); }
nb_status nb_sparse_download(const nb_field *, void *) { NB_FAIL(NB_EUNSUPPORTED, "sparse"); }
nb_status nb_sparse_fill(nb_field *, nb_fill, uint64_t, double, double) { NB_FAIL(NB_EUNSUPPORTED, "sparse"); }
nb_status nb_sparse_halo_update(nb_field *) { NB_FAIL(NB_EUNSUPPORTED, "sparse"); }
nb_status nb_sparse_axpby(double, const nb_field *, double, nb_field *, nb_view) { NB_FAIL(NB_EUNSUPPORTED, "sparse"); }
nb_status nb_sparse_dot_partials(const nb_field *, const nb_field *) { NB_FAIL(NB_EUNSUPPORTED, "sparse"); }
nb_status nb_sparse_laplace7(const nb_field *, nb_field *, nb_view) { NB_FAIL(NB_EUNSUPPORTED, "sparse"); }
nb_status nb_sparse_cg_hooks(nb_cg *, int) { NB_FAIL(NB_EUNSUPPORTED, "sparse"); }
nb_status nb_sparse_cg_init(nb_cg *) { NB_FAIL(NB_EUNSUPPORTED, "sparse"); }
nb_status nb_sparse_cg_flush(nb_cg *) { NB_FAIL(NB_EUNSUPPORTED, "sparse"); }

extern "C" nb_status nb_grid_create_sparse(const int32_t dims[3], const uint8_t *active, int32_t nparts,
                                           const int32_t *device_ids, nb_comm *comm, nb_grid **out) {
    (void)dims; (void)active; (void)nparts; (void)device_ids; (void)comm;
    if (out) *out = nullptr;
    NB_FAIL(NB_EUNSUPPORTED, "element-sparse grid not built yet");
}
