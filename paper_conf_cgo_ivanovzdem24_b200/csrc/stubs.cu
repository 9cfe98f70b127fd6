// stubs.cu -- workloads not yet implemented in this build report RODINIA_E_NOT_BUILT.
#include <vector>

#include "rg_internal.h"

namespace rg {
int srad_num_variants() { return 0; }
void srad_variant_info(int, rodinia_granularity*, const void**, const char**, int*) {}
int pathfinder_num_variants() { return 0; }
void pathfinder_variant_info(int, rodinia_granularity*, const void**, const char**, int*) {}
int lud_num_variants() { return 0; }
void lud_variant_info(int, rodinia_granularity*, const void**, const char**, int*) {}
rodinia_status tune_srad(const rodinia_problem&, int, rodinia_granularity*, std::vector<rodinia_tune_row>*) {
    return set_error(RODINIA_E_NOT_BUILT, "srad not built");
}
rodinia_status tune_pathfinder(const rodinia_problem&, int, rodinia_granularity*, std::vector<rodinia_tune_row>*) {
    return set_error(RODINIA_E_NOT_BUILT, "pathfinder not built");
}
rodinia_status tune_lud(const rodinia_problem&, int, rodinia_granularity*, std::vector<rodinia_tune_row>*) {
    return set_error(RODINIA_E_NOT_BUILT, "lud not built");
}
}  // namespace rg
