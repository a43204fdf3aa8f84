// STRICT variant: compiled with --fmad=false; bit-identical to the oracle's
// NAS evaluation order (reading c6).
#define SAFARA_STRICT_BUILD 1
#define SAFARA_VARIANT strict
// smem case table and one checked k loop: keep the STRICT kernels spill-free
#ifndef SAFARA_XREG
#define SAFARA_XREG 0
#endif
#ifndef SAFARA_PCHK_SPLIT
#define SAFARA_PCHK_SPLIT 0
#endif
#include "rhs_variant.inc"
