#include "gbtrf_window.cuh"
using namespace bandlu;
void* probes[] = {
(void*)&gbtrf_window_kernel<10,10,true,Strided<double>,Strided<int>,Strided<double>>,
(void*)&gbtrf_window_kernel<2,32,true,Strided<double>,Strided<int>,Strided<double>>,
(void*)&gbtrf_window_kernel<1,1,true,Strided<double>,Strided<int>,Strided<double>>,
(void*)&gbtrf_window_kernel<0,0,true,Strided<double>,Strided<int>,Strided<double>>,
};
