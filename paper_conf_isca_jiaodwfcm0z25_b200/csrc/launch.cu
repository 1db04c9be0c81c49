// launch.cu -- process-wide launch options.
#include <cstdlib>

#include "common.cuh"

// Programmatic dependent launch is off by default: measured on B200 it did not shorten the
// step (0.632 -> 0.637 ms with graphs and 2 streams).  NEO_PDL=1 enables it.
bool neo_pdl_enabled() {
    static const bool on = [] {
        const char* e = std::getenv("NEO_PDL");
        return e && e[0] == '1';
    }();
    return on;
}
bool neo_pdl_bconv() {
    static const bool on = [] {
        const char* e = std::getenv("NEO_PDL");
        return e && e[0] == '2';
    }();
    return on || neo_pdl_enabled();
}
