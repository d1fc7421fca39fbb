#define H1_CFG 32, kH1, 32, 16, 32, 24, 6, false
#define H2_CFG 64, kH2, 32, 16, 64, 16, 6, false
#define H6_CFG 1024, kH6, 192, 96, 384, 1, 6, true
