// Production variant: compiled with --fmad=true (FMA contraction allowed;
// parity vs the oracle within |g-o| <= 1e-12|o| + 1e-14, reading c5).
#define SAFARA_STRICT_BUILD 0
#define SAFARA_VARIANT fast
#include "rhs_variant.inc"
