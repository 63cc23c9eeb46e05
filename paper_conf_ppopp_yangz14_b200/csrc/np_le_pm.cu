// np_le_pm.cu -- the point-major instantiations of np_le.cu (LE, Figs 5-6),
// a separate translation unit only so the two layouts compile in parallel.
#define CUDANP_LE_PM_TU 1
#include "np_le.cu"
