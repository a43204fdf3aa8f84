// STRICT variant: compiled with --fmad=false; bit-identical to the oracle's
// NAS evaluation order (reading c6).
#define SAFARA_STRICT_BUILD 1
#define SAFARA_VARIANT strict
#include "rhs_variant.inc"
