"""B200-native ADADELTA energy+gradient hot path (AutoDock-GPU LS, Solis-Vasquez et al. IA3@SC'25)."""
