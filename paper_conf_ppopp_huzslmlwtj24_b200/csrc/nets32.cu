// fp32 nets (real.cuh, reading Z22): nets.cu compiled with real = float into namespace fekf::n32.
#define FEKF_NETS32 1
#include "nets.cu"
