// tb_lib.cu -- single translation unit of libtfhe_b200.so (the NTT constant banks live in one module).
#include "tb_bootstrap.cu"
#include "tb_br6.cu"
#include "tb_br9.cu"
#include "tb_brf.cu"
#include "tb_brl.cu"
#include "tb_keyswitch.cu"
#include "tb_diag.cu"
#include "tb_runtime.cu"
