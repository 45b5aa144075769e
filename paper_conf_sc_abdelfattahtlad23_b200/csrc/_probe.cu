#include "gbtrf_window.cuh"
using namespace bandlu;
void* probes[] = {
(void*)&gbtrf_window_kernel<10,10,Strided<double>,Strided<int>>,
};
