#include "gbtrf_window.cuh"
using namespace bandlu;
void* probes[] = {
(void*)&gbtrf_window_kernel<10,10,true,Strided<double>,Strided<int>,Strided<double>>,
};
