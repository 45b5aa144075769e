#include "gbtrs_window.cuh"
using namespace bandlu;
void* probes[] = {
(void*)&gbtrs_window_kernel<10,10,Strided<const double>,Strided<const int>,Strided<double>>,
(void*)&gbtrs_window_kernel<1,1,Strided<const double>,Strided<const int>,Strided<double>>,
};
