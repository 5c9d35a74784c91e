// csrc/kernels_sub.cu — the row kernels of the paper's (N/M, M, 1) block
// mapping: kernels.cu compiled with ENS_SUB=1 (see there).
#define ENS_SUB 1
#include "kernels.cu"
