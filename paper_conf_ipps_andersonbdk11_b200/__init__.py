"""B200-native (sm_100a) TSQR/CAQR: the data-parallel hot path of Anderson, Ballard,
Demmel, Keutzer, "Communication-Avoiding QR Decomposition for GPUs" (IPDPS 2011)."""
