// rtm_partition.cu - the sample partition kernels (k_partition_lm, k_partition_mx) and their
// launchers, compiled as a module of their own from rtm_kernels.cu (RTM_TU_PARTITION), in parallel
// with the rest of the library.
#define RTM_TU_PARTITION 1
#include "rtm_kernels.cu"
