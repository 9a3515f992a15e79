"""B200-native batched GATK PairHMM forward (Wang, Xie, Cong, IPDPS 2017 hot path)."""
